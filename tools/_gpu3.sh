mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_panel_gpu.py -x -q > gpurun_out/r2_panel_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_panel_tests.log
timeout 600 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --e2e-steps 5 > gpurun_out/r2_bench_band.log 2>&1; echo "rc=$?" >> gpurun_out/r2_bench_band.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"panel_kernel" -s 3 -c 1 -o gpurun_out/r2_panel_prof python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu.log 2>&1; echo "rc=$?" >> gpurun_out/r2_ncu.log
