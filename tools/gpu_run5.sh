timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests5.log 2>&1; echo "rc=$?" >> gpurun_out/gputests5.log
rm -f gpurun_out/probe5.md
timeout 600 python tools/roofline_probe.py --config c5 --iters 30 --md gpurun_out/probe5.md > gpurun_out/probe5.jsonl 2> gpurun_out/probe5.err
timeout 600 python bench.py --steps 200 --no-cpu-baseline > gpurun_out/bench5.log 2>&1
