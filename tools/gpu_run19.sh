# L2 bulk prefetch of the workgroup's next tile: C5 tpc sweep + tpc/strategy-2 parity
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,8,2,4 --iters 30 > gpurun_out/tpc19.jsonl 2> gpurun_out/tpc19.err
timeout 1500 python -m pytest tests/test_tiles_per_cta_gpu.py tests/test_strategy2_gpu.py tests/test_spmv_gpu.py -q > gpurun_out/gputests19.log 2>&1; echo "rc=$?" >> gpurun_out/gputests19.log
