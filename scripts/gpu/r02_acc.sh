mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -k "accumulate or subnormal or late_join or c3_ or tma_large" > gpurun_out/t2_focus.log 2>&1; echo "focus rc=$?" >> gpurun_out/t2_focus.log
timeout 600 python scripts/bench_accumulate.py --out gpurun_out/acc_r02_a.json > gpurun_out/t2_acc.log 2>&1; echo "acc rc=$?" >> gpurun_out/t2_acc.log
