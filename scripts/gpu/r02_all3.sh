mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q --timeout 300 -k "ddp or aliased" > gpurun_out/t13_ddp.log 2>&1; echo "rc=$?" >> gpurun_out/t13_ddp.log
timeout 1800 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/t13_all.log 2>&1; echo "rc=$?" >> gpurun_out/t13_all.log
