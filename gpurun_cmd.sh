python scripts/debug/ab_configs.py --coll allreduce --sizes 10,16,18,20,21,22 --reps 5 --configs 'engine=2;sched=0' 2>&1 | tail -6
python scripts/debug/ab_configs.py --coll alltoall --sizes 10,20,22 --reps 5 --configs 'engine=2' 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
