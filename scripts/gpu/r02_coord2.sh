mkdir -p gpurun_out
python -m paper_conf_icdcs_zhaozw24_b200._build > gpurun_out/t11_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q --timeout 300 -k "coordinator or ddp or fault or exclu" > gpurun_out/t11_coord.log 2>&1; echo "rc=$?" >> gpurun_out/t11_coord.log
timeout 1200 python scripts/bench_c3.py --out gpurun_out/c3_r02b.json > gpurun_out/t11_c3.log 2>&1; echo "rc=$?" >> gpurun_out/t11_c3.log
