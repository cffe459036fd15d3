bash scripts/profile.sh r01 > gpurun_out/profile_run.log 2>&1
python scripts/sweep_sizes.py --graph --out gpurun_out/sizes_ar.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --coll alltoall --out gpurun_out/sizes_a2a.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --coll allgather --out gpurun_out/sizes_ag.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --dtype bf16 --out gpurun_out/sizes_ar_bf16.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/debug/launch_floor.py > gpurun_out/floor.json 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
tail -1 gpurun_out/bench_r01.json | cut -c1-200; cat gpurun_out/smoke.log
