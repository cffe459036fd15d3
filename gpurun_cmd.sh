python scripts/debug/ab_configs.py --coll allreduce --sizes 10,16,20,21,22,23,24,25 --reps 5 --configs 'engine=2;engine=1;engine=0' 2>&1 | tail -8
python scripts/debug/ab_configs.py --coll alltoall --sizes 10,20,22,23,24 --reps 5 --configs 'engine=2' 2>&1 | tail -5
for s in 1048576 4194304; do python scripts/trace_report.py --bytes-per-rank $s --out gpurun_out/tr/b_ar_$s > /dev/null 2>gpurun_out/tr/err_$s.log; done
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/t_all.log 2>&1; tail -2 gpurun_out/t_all.log
