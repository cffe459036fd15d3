cd paper_conf_icdcs_zhaozw24_b200
for r in 1 2; do
 for v in u1 u2; do
  cp lib_$v.so.ab libadapcc.so
  (cd .. && python scripts/bench_accumulate.py --sizes 1,4,16,25,64,100 --variants red:0,flat:0 > gpurun_out/acc_flat_$v.$r.log 2>&1)
 done
done
cp lib_u2.so.ab libadapcc.so
cd .. && ADAPCC_ENGINE=3 timeout 900 python -m pytest tests/test_gpu_loopback.py tests/test_gpu_primitives.py tests/test_gpu_fuzz.py tests/test_gpu_ipc_zerocopy.py -m gpu -q > gpurun_out/flat_u2_tests.log 2>&1; tail -2 gpurun_out/flat_u2_tests.log
