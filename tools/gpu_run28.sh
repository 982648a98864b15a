# non-finite propagation tests (NaN values, Inf x) on the committed build
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_nonfinite_gpu.py -q > gpurun_out/gputests28.log 2>&1; echo "rc=$?" >> gpurun_out/gputests28.log
