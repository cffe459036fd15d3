mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:flat -s 3 -c 1 -o gpurun_out/prof_acc1_flat_r02b python scripts/debug/acc_one.py 1 1 > gpurun_out/ncu_acc1_flat.log 2>&1
ADAPCC_ENGINE=3 ncu --set full --clock-control none --import-source on -k regex:flat -s 3 -c 1 -o gpurun_out/prof_acc16_flat_r02b python scripts/debug/acc_one.py 16 1 > gpurun_out/ncu_acc16_flat.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:engine -s 3 -c 1 -o gpurun_out/prof_acc16_red1_r02b python scripts/debug/acc_one.py 16 1 > gpurun_out/ncu_acc16_red.log 2>&1
ls -la gpurun_out
