mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -x -k "racing or subnormal or interleaved" > gpurun_out/t4_focus.log 2>&1; echo "focus rc=$?" >> gpurun_out/t4_focus.log
timeout 300 python scripts/bench_accumulate.py --variants red:0,rmw:0 --out gpurun_out/acc_r02.json > gpurun_out/t4_acc.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/t4_all.log 2>&1; echo "all rc=$?" >> gpurun_out/t4_all.log
