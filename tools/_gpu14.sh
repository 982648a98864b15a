mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_panel_gpu.py -x -q > gpurun_out/r2_panel_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_panel_tests.log
rm -f gpurun_out/r2_sweep15.log
for P in '{}' '{"S":1}' '{"S":3}' '{"S":4}'; do
  echo "== $P" >> gpurun_out/r2_sweep15.log
  timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 --params "$P" 2>&1 | grep -o '"ms_per_step": [0-9.]*\|"kernels": {[^}]*}[^}]*}[^}]*}\|Error.*' >> gpurun_out/r2_sweep15.log
done
