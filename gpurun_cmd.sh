python scripts/debug/ab_configs.py --coll allgather --sizes 23,24,25,26 --reps 5 --configs 'engine=0;engine=1;engine=0,sched=0' 2>&1 | tail -4
python scripts/debug/ab_configs.py --coll allreduce --sizes 23,24,25 --reps 5 --configs 'engine=0;engine=1' 2>&1 | tail -3
python scripts/debug/ab_configs.py --coll alltoall --sizes 23,24,25 --reps 5 --configs 'engine=0;engine=1' 2>&1 | tail -3
