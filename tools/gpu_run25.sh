# Fig. 14 ablation with the current kernel (tiles_per_cta auto) + tuned-vs-exhaustive configs
timeout 1500 python tools/ablation.py --md gpurun_out/ablation25.md > gpurun_out/ablation25.jsonl 2> gpurun_out/ablation25.err
timeout 1500 python tools/bench_configs.py --exhaustive --md gpurun_out/configs25.md > gpurun_out/configs25.jsonl 2> gpurun_out/configs25.err
