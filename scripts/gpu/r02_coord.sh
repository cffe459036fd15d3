mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -k "coordinator" > gpurun_out/t8_coord.log 2>&1; echo "rc=$?" >> gpurun_out/t8_coord.log
timeout 1200 python scripts/bench_c3.py --out gpurun_out/c3_r02.json > gpurun_out/t8_c3.log 2>&1; echo "rc=$?" >> gpurun_out/t8_c3.log
