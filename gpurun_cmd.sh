bash scripts/profile.sh r01 > gpurun_out/profile_run.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
tail -1 gpurun_out/bench_r01.json | cut -c1-160; cat gpurun_out/smoke.log
