rm -f gpurun_out/probe_sweep.md
timeout 900 python tools/roofline_probe.py --config c5 --iters 20 --md gpurun_out/probe_sweep.md --sweep '{}' '{"T":32,"C":64}' '{"T":32,"C":256}' '{"T":16,"C":128}' '{"T":16,"C":256}' > gpurun_out/probe_sweep.jsonl 2> gpurun_out/probe_sweep.err
