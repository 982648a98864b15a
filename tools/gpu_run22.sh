# final round-1 verification of the committed build: GPU suite, smoke, default bench
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/gputests22.log 2>&1; echo "rc=$?" >> gpurun_out/gputests22.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke22.log 2>&1; echo "rc=$?" >> gpurun_out/smoke22.log
timeout 900 python bench.py > gpurun_out/bench22.log 2>&1; echo "rc=$?" >> gpurun_out/bench22.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench22_ref.log 2>&1; echo "rc=$?" >> gpurun_out/bench22_ref.log
