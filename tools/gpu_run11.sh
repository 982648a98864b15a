# e2e with 3 host slots (bench), DRAM/L2/L1 traffic of each roofline probe (ncu), GPU tests
timeout 900 python bench.py --no-cpu-baseline --e2e-steps 40 > gpurun_out/bench11.log 2>&1; echo "rc=$?" >> gpurun_out/bench11.log
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:spmv_bccoo --csv --log-file gpurun_out/probe_traffic11.csv python tools/roofline_probe.py --config c5 --ncu > gpurun_out/probe_traffic11.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gputests11.log 2>&1; echo "rc=$?" >> gpurun_out/gputests11.log
