# final check of HEAD: whole GPU suite (incl. test_nonfinite_gpu.py) and smoke
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/gputests29.log 2>&1; echo "rc=$?" >> gpurun_out/gputests29.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke29.log 2>&1; echo "rc=$?" >> gpurun_out/smoke29.log
