timeout 1200 python -m pytest tests/test_fused_gpu.py tests/test_dist_gpu.py -q > gpurun_out/gputests24.log 2>&1; echo "rc=$?" >> gpurun_out/gputests24.log
