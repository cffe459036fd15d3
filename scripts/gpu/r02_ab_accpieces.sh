cd paper_conf_icdcs_zhaozw24_b200
for r in 1 2; do
 for v in old new; do
  cp lib_$v.so.ab libadapcc.so
  (cd .. && python scripts/bench_accumulate.py --sizes 16,25,64,100,256 --variants red:0 > gpurun_out/acc_ab_$v.$r.log 2>&1)
 done
done
cp lib_new.so.ab libadapcc.so
cd .. && timeout 900 python -m pytest tests/test_gpu_loopback.py tests/test_gpu_fullsize.py tests/test_gpu_fuzz.py -m gpu -q -k "accumulate or c3 or fuzz" > gpurun_out/accpieces_tests.log 2>&1; tail -2 gpurun_out/accpieces_tests.log
