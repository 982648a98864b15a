# GPU suite; ncu (full + launch list) of the tiles_per_cta = 2 kernel, summarised on the box (the .ncu-rep stays behind)
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputests16.log 2>&1; echo "rc=$?" >> gpurun_out/gputests16.log
mkdir -p /tmp/ncu16
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:spmv_bccoo -s 2 -c 1 -o /tmp/ncu16/c5_full python tools/profile_spmv.py --config c5 --params '{"T":32,"C":128,"col_mode":2}' --iters 3 > gpurun_out/ncu_full16.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches16.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_ncu16.log 2>&1
python tools/ncu_summary.py --rep /tmp/ncu16/c5_full.ncu-rep --alg-bytes 8551758880 --out gpurun_out/r01_c5_spmv16 --title "Round 1 (tiles_per_cta = 2) — C5 (50M rows, 1.0B nnz, fp32), spmv_bccoo_kernel<float,1,1,32,I32>, C=128; ncu --set full --clock-control none" > gpurun_out/summ16.log 2>&1
ncu -i /tmp/ncu16/c5_full.ncu-rep --page details --csv > gpurun_out/c5_full16_details.csv 2>/dev/null
timeout 900 python bench.py --params '{"S":2}' --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench16_s2.log 2>&1
timeout 900 python bench.py --params '{"tpc":4}' --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench16_tpc4.log 2>&1
du -sh gpurun_out >> gpurun_out/summ16.log
