# GPU suite after the reencode keep-current fix; ncu (full + launch list) of the tiles_per_cta = 2 kernel
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputests15.log 2>&1; echo "rc=$?" >> gpurun_out/gputests15.log
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmv_bccoo -s 2 -c 1 -o gpurun_out/c5_full15 python tools/profile_spmv.py --config c5 --params '{"T":32,"C":128,"col_mode":2}' --iters 3 > gpurun_out/ncu_full15.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches15.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_ncu15.log 2>&1
