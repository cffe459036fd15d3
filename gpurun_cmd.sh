timeout 900 python scripts/bench_configs.py --only C4v --out gpurun_out/configs_c4v.json 2>&1 | tail -5
