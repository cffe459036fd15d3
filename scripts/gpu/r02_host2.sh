mkdir -p gpurun_out
bash scripts/debug/host_floor.sh > gpurun_out/host_floor3.log 2>&1
bash scripts/gpu/r02_host.sh
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/t5_all.log 2>&1; echo "all rc=$?" >> gpurun_out/t5_all.log
