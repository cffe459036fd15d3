timeout 600 python -m pytest tests/test_gpu_late_join.py -x -q -p no:cacheprovider -k graph 2>&1 | tail -15
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
