mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -rs --timeout 300 -k "nvls" > gpurun_out/t11_nvls.log 2>&1; echo "rc=$?" >> gpurun_out/t11_nvls.log
