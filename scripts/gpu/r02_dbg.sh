mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ipc_late.py tests/test_gpu_coordinator.py -q --timeout 600 -k "after_exclusion or fault" > gpurun_out/t12.log 2>&1; echo "rc=$?" >> gpurun_out/t12.log
