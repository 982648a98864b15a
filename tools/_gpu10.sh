mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_panel_gpu.py -x -q > gpurun_out/r2_panel_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_panel_tests.log
timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 > gpurun_out/r2_bench10.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"panel_kernel" -s 3 -c 1 -o /tmp/p10 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu10.log 2>&1
ncu -i /tmp/p10.ncu-rep --page raw --csv > gpurun_out/r2_panel10_raw.csv 2>/dev/null
ncu -i /tmp/p10.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/r2_panel10_src.csv 2>/dev/null
timeout 900 ncu --section MemoryWorkloadAnalysis --section SpeedOfLight --metrics lts__t_sector_hit_rate.pct,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum --clock-control none -k regex:"spmv_bccoo|combine" -s 4 -c 2 -o /tmp/f10 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 --params '{"S":2}' > gpurun_out/r2_ncu10f.log 2>&1
ncu -i /tmp/f10.ncu-rep --page raw --csv > gpurun_out/r2_far10_s2_raw.csv 2>/dev/null
