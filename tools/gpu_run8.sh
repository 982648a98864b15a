timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests8.log 2>&1; echo "rc=$?" >> gpurun_out/gputests8.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke8.log 2>&1; echo "rc=$?" >> gpurun_out/smoke8.log
rm -f gpurun_out/probe8.md
timeout 600 python tools/roofline_probe.py --config c5 --iters 30 --md gpurun_out/probe8.md > gpurun_out/probe8.jsonl 2> gpurun_out/probe8.err
timeout 900 python bench.py > gpurun_out/bench8.log 2>&1; echo "rc=$?" >> gpurun_out/bench8.log
