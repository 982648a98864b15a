mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_panel_gpu.py -x -q > gpurun_out/r2_panel_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2_panel_tests.log
rm -f gpurun_out/r2_sweep5.log
for P in '{}' '{"rc":1}' '{"rc":2}' '{"rc":1,"T":16,"C":256}'; do
  echo "== $P" >> gpurun_out/r2_sweep5.log
  timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --e2e-steps 2 --params "$P" 2>&1 | grep -o '"ms_per_step": [0-9.]*\|"kernels": {[^}]*}[^}]*}[^}]*}\|Error.*' >> gpurun_out/r2_sweep5.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"panel_kernel" -s 3 -c 1 -o gpurun_out/r2_panel_prof2 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu2.log 2>&1; echo "rc=$?" >> gpurun_out/r2_ncu2.log
