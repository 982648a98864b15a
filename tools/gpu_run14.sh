# tiles_per_cta as a parameter: full GPU suite, smoke, bench (default), C5 tpc sweep, configs (tuner incl. tpc)
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputests14.log 2>&1; echo "rc=$?" >> gpurun_out/gputests14.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke14.log 2>&1; echo "rc=$?" >> gpurun_out/smoke14.log
timeout 900 python bench.py > gpurun_out/bench14.log 2>&1; echo "rc=$?" >> gpurun_out/bench14.log
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,1,2,4 --iters 30 > gpurun_out/tpc14.jsonl 2> gpurun_out/tpc14.err
timeout 900 python tools/bench_configs.py --md gpurun_out/configs14.md > gpurun_out/configs14.jsonl 2> gpurun_out/configs14.err
