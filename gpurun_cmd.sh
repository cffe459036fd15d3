python scripts/debug/acc_engines.py 2>&1 | tail -4
python scripts/debug/late_timing.py 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_late_join.py tests/test_gpu_fuzz.py tests/test_gpu_loopback.py tests/test_gpu_primitives.py -x -q -p no:cacheprovider 2>&1 | tail -2
