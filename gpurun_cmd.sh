timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
python scripts/debug/late_timing.py 2>&1 | tail -1
