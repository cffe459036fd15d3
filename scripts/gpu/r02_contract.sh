mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_bench_contract.py -q -m gpu --timeout 900 > gpurun_out/t10_contract.log 2>&1; echo "rc=$?" >> gpurun_out/t10_contract.log
timeout 600 python bench.py --gpus 2 --test-same-gpu --steps 3 --warmup 3 --size-mib 8 --e2e-steps 2 --no-sweep > gpurun_out/t10_same.json 2> gpurun_out/t10_same.err; echo "rc=$?" >> gpurun_out/t10_same.err
