# in-workgroup successors skip the hand-off exchange: C5 tpc sweep + carry/tpc/fused parity
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,2,4 --iters 30 > gpurun_out/tpc23.jsonl 2> gpurun_out/tpc23.err
timeout 1800 python -m pytest tests/test_tiles_per_cta_gpu.py tests/test_spmv_gpu.py tests/test_strategy2_gpu.py tests/test_fused_gpu.py tests/test_c5_full_gpu.py tests/test_runtime_gpu.py -q > gpurun_out/gputests23.log 2>&1; echo "rc=$?" >> gpurun_out/gputests23.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench23.log 2>&1; echo "rc=$?" >> gpurun_out/bench23.log
