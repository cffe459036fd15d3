python scripts/debug/ab_configs.py --coll allreduce --sizes 10,16,20,22,23,24,25 --reps 5 --configs 'engine=2;engine=1' 2>&1 | tail -7
python scripts/debug/ab_configs.py --coll alltoall --sizes 10,20,23,24 --reps 5 --configs 'engine=2;engine=1' 2>&1 | tail -4
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
