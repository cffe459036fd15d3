mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 300 > gpurun_out/t15_all.log 2>&1; echo "rc=$?" >> gpurun_out/t15_all.log
timeout 900 python bench.py > gpurun_out/t15_bench.json 2> gpurun_out/t15_bench.err; echo "rc=$?" >> gpurun_out/t15_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/t15_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/t15_smoke.log
