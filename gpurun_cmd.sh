ncu --set full --clock-control none -k regex:engine -s 2 -c 1 -o gpurun_out/prof_acc16 python scripts/debug/acc_one.py > gpurun_out/ncu_acc.log 2>&1; tail -2 gpurun_out/ncu_acc.log
