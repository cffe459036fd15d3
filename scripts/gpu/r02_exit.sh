mkdir -p gpurun_out
timeout 1500 python scripts/debug/exit_ab.py --rounds 3 > gpurun_out/exit_ab.log 2>&1; echo "rc=$?" >> gpurun_out/exit_ab.log
