mkdir -p gpurun_out
python -m paper_conf_icdcs_zhaozw24_b200._build > gpurun_out/t9_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 -k "coordinator_fault" > gpurun_out/t9_fault.log 2>&1; echo "rc=$?" >> gpurun_out/t9_fault.log
