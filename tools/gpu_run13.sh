# tiles-per-CTA without the inter-tile barrier (double-buffered scan state): C5 / C4 / C3 timing + parity under TPC=2,4
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,3,4,8,1 > gpurun_out/tpc13.jsonl 2> gpurun_out/tpc13.err
timeout 600 python tools/tpc_sweep.py --config c5 --rc 1 --tpc 1,2,4 >> gpurun_out/tpc13.jsonl 2>> gpurun_out/tpc13.err
timeout 600 python tools/tpc_sweep.py --config c4 --params '{"T":16,"C":128,"col_mode":2}' --tpc 1,2,4,1 --iters 50 >> gpurun_out/tpc13.jsonl 2>> gpurun_out/tpc13.err
timeout 600 python tools/tpc_sweep.py --config c3-ship --params '{"h":2,"w":2,"T":16,"C":256,"col_mode":3}' --tpc 1,2,4,1 --iters 50 >> gpurun_out/tpc13.jsonl 2>> gpurun_out/tpc13.err
YASPMV_TILES_PER_CTA=2 timeout 1200 python -m pytest tests/test_spmv_gpu.py tests/test_strategy2_gpu.py tests/test_runtime_gpu.py tests/test_fused_gpu.py -x -q > gpurun_out/tpc_tests13a.log 2>&1; echo "rc=$?" >> gpurun_out/tpc_tests13a.log
YASPMV_TILES_PER_CTA=3 timeout 1200 python -m pytest tests/test_spmv_gpu.py tests/test_strategy2_gpu.py -x -q > gpurun_out/tpc_tests13b.log 2>&1; echo "rc=$?" >> gpurun_out/tpc_tests13b.log
