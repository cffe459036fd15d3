mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/s2_smi.log
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/s2_all.log 2>&1; echo "all rc=$?" >> gpurun_out/s2_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s2_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/s2_smoke.log
timeout 600 python bench.py > gpurun_out/s2_bench.json 2> gpurun_out/s2_bench.err; echo "bench rc=$?" >> gpurun_out/s2_bench.err
