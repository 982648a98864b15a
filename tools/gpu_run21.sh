# 80-register cap (6 CTAs/SM, with spills) for the fp32 scalar instances: C5 tpc sweep
timeout 900 python tools/tpc_sweep.py --config c5 --tpc 1,2,4,2 --iters 30 > gpurun_out/tpc21.jsonl 2> gpurun_out/tpc21.err
