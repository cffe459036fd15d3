timeout 900 python scripts/bench_configs.py --only C3 --out gpurun_out/configs_c3.json > gpurun_out/c3.log 2>&1; tail -1 gpurun_out/c3.log | cut -c1-100
timeout 900 python scripts/bench_configs.py --only C3 --out gpurun_out/configs_c3b.json > gpurun_out/c3b.log 2>&1; tail -1 gpurun_out/c3b.log | cut -c1-100
