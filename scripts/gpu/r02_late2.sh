mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -k "late or coordinator" > gpurun_out/t12_late.log 2>&1; echo "rc=$?" >> gpurun_out/t12_late.log
timeout 1200 python scripts/bench_c3.py --out gpurun_out/c3_r02b.json > gpurun_out/t12_c3.log 2>&1; echo "rc=$?" >> gpurun_out/t12_c3.log
