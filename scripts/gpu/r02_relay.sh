mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q --timeout 300 -k "relay_store or wide_rank" > gpurun_out/t10_relay.log 2>&1; echo "rc=$?" >> gpurun_out/t10_relay.log
timeout 900 python scripts/bench_relay.py --out gpurun_out/relay_ab_r02.json > gpurun_out/t10_relay_ab.log 2>&1; echo "rc=$?" >> gpurun_out/t10_relay_ab.log
timeout 900 python bench.py --gpus 2 --test-same-gpu --steps 5 --warmup 3 --size-mib 16 --e2e-steps 2 > gpurun_out/t10_multi.json 2> gpurun_out/t10_multi.err; echo "rc=$?" >> gpurun_out/t10_multi.err
