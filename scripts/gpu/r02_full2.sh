mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q --timeout 200 -k "nvls" > gpurun_out/t9_nvls.log 2>&1; echo "rc=$?" >> gpurun_out/t9_nvls.log
timeout 1800 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/t9_all.log 2>&1; echo "rc=$?" >> gpurun_out/t9_all.log
