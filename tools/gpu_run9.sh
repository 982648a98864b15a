# C5 slice sweep + ncu launch list of the bench + one --set full capture of K1 (round 1, after the non-blocking carries)
timeout 900 python tools/sweep.py --config c5 --iters 20 --sets '[{"T":32,"C":128,"col_mode":2,"S":1},{"T":32,"C":128,"col_mode":2,"S":2},{"T":32,"C":128,"col_mode":2,"S":4},{"T":32,"C":128,"col_mode":2,"S":8},{"T":16,"C":256,"col_mode":2,"S":1},{"T":32,"C":128,"col_mode":3,"S":1}]' > gpurun_out/sweep9.jsonl 2> gpurun_out/sweep9.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches9.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_ncu9.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmv_bccoo -s 2 -c 1 -o gpurun_out/c5_full9 python tools/profile_spmv.py --config c5 --params '{"T":32,"C":128,"col_mode":2}' --iters 3 > gpurun_out/ncu_full9.log 2>&1
ls -la gpurun_out >> gpurun_out/ncu_full9.log
