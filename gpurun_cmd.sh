bash scripts/sanitize.sh > /dev/null 2>&1; grep -h "== exit\|ERROR SUMMARY\|RACECHECK SUMMARY\|passed\|failed" gpurun_out/sanitize_*.log
grep -E "Error: Race" gpurun_out/sanitize_racecheck.log | sed -E 's/\+0x[0-9a-f]+//g; s/\(.*\)//' | sort | uniq -c | head
timeout 900 python -m pytest tests/test_gpu_late_join.py tests/test_gpu_loopback.py -x -q -p no:cacheprovider 2>&1 | tail -1
