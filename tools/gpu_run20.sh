# streaming (evict-first) y stores: C5 tpc sweep, sustained bench, parity
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,2 --iters 30 > gpurun_out/tpc20.jsonl 2> gpurun_out/tpc20.err
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench20.log 2>&1; echo "rc=$?" >> gpurun_out/bench20.log
timeout 1500 python -m pytest tests/test_tiles_per_cta_gpu.py tests/test_spmv_gpu.py tests/test_fused_gpu.py -q > gpurun_out/gputests20.log 2>&1; echo "rc=$?" >> gpurun_out/gputests20.log
