mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_panel_gpu.py -x -q > gpurun_out/r2_panel_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_panel_tests.log
timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 > gpurun_out/r2_bench13.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"panel_kernel" -s 3 -c 1 -o /tmp/p13 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu13.log 2>&1
ncu -i /tmp/p13.ncu-rep --page raw --csv > gpurun_out/r2_panel13_raw.csv 2>/dev/null
ncu -i /tmp/p13.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/r2_panel13_src.csv 2>/dev/null
