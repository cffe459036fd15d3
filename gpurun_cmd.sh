timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
timeout 300 python bench.py > gpurun_out/bench2.json 2> gpurun_out/bench2.err
python scripts/sweep_sizes.py --graph --out gpurun_out/sizes_ar_r01b.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --coll alltoall --out gpurun_out/sizes_a2a_r01b.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --coll allgather --out gpurun_out/sizes_ag_r01b.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/sweep_sizes.py --graph --dtype bf16 --out gpurun_out/sizes_ar_bf16_r01b.json > /dev/null 2>>gpurun_out/st_err.log
python scripts/debug/launch_floor.py > gpurun_out/floor3.json 2>&1
