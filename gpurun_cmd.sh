timeout 600 python -m pytest tests/test_gpu_ddp_hook.py -q -p no:cacheprovider > gpurun_out/t_ddp.log 2>&1; tail -15 gpurun_out/t_ddp.log
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
