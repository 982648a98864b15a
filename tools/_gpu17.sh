mkdir -p gpurun_out
rm -f gpurun_out/r2_sweep17.log
for P in '{"R":8192,"W":8192}' '{"R":8192,"W":8192,"S":2}' '{"R":8192,"W":6144}'; do
  echo "== $P" >> gpurun_out/r2_sweep17.log
  timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 --params "$P" 2>&1 | grep -o '"ms_per_step": [0-9.]*\|"kernels": {[^}]*}[^}]*}[^}]*}\|Error.*' >> gpurun_out/r2_sweep17.log
done
