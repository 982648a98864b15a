# tiles-per-CTA experiment + store-tail probes (10, 11) + GPU tests
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,8,16,1 > gpurun_out/tpc12.jsonl 2> gpurun_out/tpc12.err
timeout 600 python tools/tpc_sweep.py --config c4 --params '{"T":16,"C":128,"col_mode":2}' --tpc 1,2,4,1 --iters 50 >> gpurun_out/tpc12.jsonl 2>> gpurun_out/tpc12.err
rm -f gpurun_out/probe12.md
timeout 600 python tools/roofline_probe.py --config c5 --iters 20 --md gpurun_out/probe12.md > gpurun_out/probe12.jsonl 2> gpurun_out/probe12.err
YASPMV_TILES_PER_CTA=4 timeout 1200 python -m pytest tests/test_spmv_gpu.py tests/test_strategy2_gpu.py -x -q > gpurun_out/tpc_tests12.log 2>&1; echo "rc=$?" >> gpurun_out/tpc_tests12.log
