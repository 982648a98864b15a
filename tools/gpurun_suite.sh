#!/bin/bash
# One parameterised GPU-box runner (replaces the round-1 one-off lease scripts):
#   bash tools/gpurun_suite.sh TAG STEP...   with STEP in
#     tests      pytest -m gpu (whole GPU suite)            -> gpurun_out/TAG_gputests.log
#     smoke      __graft_entry__.smoke()                   -> gpurun_out/TAG_smoke.log
#     bench      python bench.py (defaults)                -> gpurun_out/TAG_bench.log
#     ref        python bench.py --impl reference          -> gpurun_out/TAG_ref.log
#     launches   ncu launch list of a short bench          -> gpurun_out/TAG_launches.csv
#     ncu        ncu --set full of one step's band + far kernels: raw page CSV, source page of the
#                band kernel (the .ncu-rep stays on the box)  -> gpurun_out/TAG_raw.csv, TAG_src.csv
# Extra bench arguments: BENCH_ARGS="..." in the environment.
set -u
TAG=$1; shift
mkdir -p gpurun_out
for step in "$@"; do
  case $step in
    tests)  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_gputests.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_gputests.log ;;
    smoke)  timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_smoke.log ;;
    bench)  timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/${TAG}_bench.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_bench.log ;;
    ref)    timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/${TAG}_ref.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_ref.log ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
                --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline \
                --e2e-steps 2 ${BENCH_ARGS:-} > gpurun_out/${TAG}_launches.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_launches.log ;;
    ncu)    timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"panel_kernel|spmv_bccoo" \
                -s 8 -c 2 -o /tmp/${TAG}_prof python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
                --e2e-steps 1 ${BENCH_ARGS:-} > gpurun_out/${TAG}_ncu.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_ncu.log
            ncu -i /tmp/${TAG}_prof.ncu-rep --page raw --csv > gpurun_out/${TAG}_raw.csv 2>/dev/null
            ncu -i /tmp/${TAG}_prof.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>/dev/null
            ncu -i /tmp/${TAG}_prof.ncu-rep --page source --csv --print-source cuda,sass -k regex:panel_kernel \
                > gpurun_out/${TAG}_src.csv 2>/dev/null ;;
    *) echo "unknown step $step" ;;
  esac
done
