python scripts/debug/ab_configs.py --coll allreduce --sizes 23,24,25 --reps 5 --configs 'taper=0;taper=1' 2>&1 | tail -3
python scripts/debug/ab_configs.py --coll allgather --sizes 24,25 --reps 5 --configs 'taper=0;taper=1' 2>&1 | tail -2
