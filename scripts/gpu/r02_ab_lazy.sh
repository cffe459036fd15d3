cd paper_conf_icdcs_zhaozw24_b200
for r in 1 2 3; do
 for v in old new; do
  cp lib_$v.so.ab libadapcc.so
  (cd .. && python bench.py --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1 --steps 40 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'])")
 done
done
for v in old new; do cp lib_$v.so.ab libadapcc.so; (cd .. && python scripts/sweep_sizes.py --graph --min-log2 20 --max-log2 26 --out gpurun_out/sizes_lz_$v.json > /dev/null 2>&1; python scripts/bench_accumulate.py --sizes 16,25,64 --variants red:0 > gpurun_out/acc_lz_$v.log 2>&1); done
for v in old new; do cp lib_$v.so.ab libadapcc.so; (cd .. && python scripts/sweep_sizes.py --graph --min-log2 20 --max-log2 26 --out gpurun_out/sizes_lz2_$v.json > /dev/null 2>&1; python scripts/bench_accumulate.py --sizes 16,25,64 --variants red:0 > gpurun_out/acc_lz2_$v.log 2>&1); done
cp lib_new.so.ab libadapcc.so
