cd paper_conf_icdcs_zhaozw24_b200
for r in 1 2 3; do
 for v in old new start; do
  cp lib_$v.so.ab libadapcc.so
  (cd .. && python bench.py --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1 --steps 40 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', d['value'], d['ms_per_step'])")
 done
done
