mkdir -p gpurun_out
for v in main nomaxnreg lane0 both; do
  lib=paper_conf_icdcs_zhaozw24_b200/libadapcc.so; [ $v != main ] && lib=build/lib_$v.so
  echo "== $v" >> gpurun_out/t3_acc.log
  ADAPCC_LIB=$lib timeout 300 python scripts/bench_accumulate.py --sizes 16,64 --variants red:0,red:2,rmw:2 >> gpurun_out/t3_acc.log 2>&1
done
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -x -k "accumulate or subnormal or late_join or c3_ or tma_large" > gpurun_out/t3_focus.log 2>&1; echo "focus rc=$?" >> gpurun_out/t3_focus.log
