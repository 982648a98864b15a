# round-1 re-verification after the container rebuild: GPU suite, smoke, default bench, reference arm, bench launch list
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/gputests26.log 2>&1; echo "rc=$?" >> gpurun_out/gputests26.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke26.log 2>&1; echo "rc=$?" >> gpurun_out/smoke26.log
timeout 900 python bench.py > gpurun_out/bench26.log 2>&1; echo "rc=$?" >> gpurun_out/bench26.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench26_ref.log 2>&1; echo "rc=$?" >> gpurun_out/bench26_ref.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches26.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu26.log 2>&1; echo "rc=$?" >> gpurun_out/ncu26.log
