python scripts/debug/late_timing.py 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_late_join.py tests/test_gpu_fuzz.py -x -q -p no:cacheprovider 2>&1 | tail -2
