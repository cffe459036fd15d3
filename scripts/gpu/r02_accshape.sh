mkdir -p gpurun_out
for v in main d4x48 d6x32 d2x96; do
  lib=paper_conf_icdcs_zhaozw24_b200/libadapcc.so; [ $v != main ] && lib=build/lib_$v.so
  echo "== $v" >> gpurun_out/accshape.log
  ADAPCC_LIB=$lib timeout 300 python scripts/bench_accumulate.py --sizes 16,25,64 --variants red:1 >> gpurun_out/accshape.log 2>&1
done
