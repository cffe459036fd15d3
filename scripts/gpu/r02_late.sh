mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 -x -k "late" > gpurun_out/t7_late.log 2>&1; echo "rc=$?" >> gpurun_out/t7_late.log
