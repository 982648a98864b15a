mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none -k regex:"spmv_bccoo" -s 3 -c 1 -o gpurun_out/r2_far_s1 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2_ncu_far1.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"spmv_bccoo" -s 3 -c 1 -o gpurun_out/r2_far_s4 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 --params '{"S":4}' > gpurun_out/r2_ncu_far4.log 2>&1
