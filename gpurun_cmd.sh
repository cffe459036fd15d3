timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
timeout 1200 python scripts/bench_configs.py --out gpurun_out/configs_new.json > gpurun_out/configs_new.log 2>&1; tail -3 gpurun_out/configs_new.log
python scripts/debug/host_overhead.py > gpurun_out/host_overhead.txt 2>&1
