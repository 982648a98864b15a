mkdir -p gpurun_out
for P in '{"S":2}' '{"S":4}' '{"T":16,"C":256}' '{"S":4,"T":16,"C":256}'; do
  echo "== $P" >> gpurun_out/r2_far_sweep.log
  timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 --params "$P" 2>&1 | grep -o '"ms_per_step": [0-9.]*\|"kernels": {[^}]*}[^}]*}[^}]*}' >> gpurun_out/r2_far_sweep.log
done
