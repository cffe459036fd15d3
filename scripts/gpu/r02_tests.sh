set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -x -k "late_join or fullsize or zero_copy or bench_contract" > gpurun_out/t1_focus.log 2>&1; echo "focus rc=$?" >> gpurun_out/t1_focus.log
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/t1_all.log 2>&1; echo "all rc=$?" >> gpurun_out/t1_all.log
timeout 600 python bench.py > gpurun_out/t1_bench.json 2> gpurun_out/t1_bench.err; echo "bench rc=$?" >> gpurun_out/t1_bench.err
