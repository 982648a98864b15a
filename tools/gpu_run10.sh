# strategy 2 (result cache) parity + full GPU suite + C5 s1/s2 timing
timeout 900 python -m pytest tests/test_strategy2_gpu.py -x -q > gpurun_out/s2tests10.log 2>&1; echo "rc=$?" >> gpurun_out/s2tests10.log
timeout 900 python tools/sweep.py --config c5 --iters 20 --sets '[{"T":32,"C":128,"col_mode":2},{"T":32,"C":128,"col_mode":2,"rc":1},{"T":32,"C":128,"col_mode":2,"rc":2},{"T":16,"C":256,"col_mode":2,"rc":1}]' > gpurun_out/sweep10.jsonl 2> gpurun_out/sweep10.err
timeout 900 python tools/bench_configs.py --md gpurun_out/configs10.md > gpurun_out/configs10.jsonl 2> gpurun_out/configs10.err
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests10.log 2>&1; echo "rc=$?" >> gpurun_out/gputests10.log
