#!/bin/bash
# Round-2 GPU-box profiling (B200_PROFILING.md recipe): bench line, launch list,
# one ncu --set full capture per kernel of interest, host-overhead probe.
# Usage (under gpurun): bash scripts/profile_r02.sh <tag>
set -u
TAG=${1:-r02}
OUT=gpurun_out
mkdir -p $OUT
python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1 > /dev/null 2>&1
SHORT="--steps 3 --warmup 3 --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1"
for cfg in "direct 1" "staged 1"; do
  set -- $cfg
  name=${1}_$([ $2 = 1 ] && echo tma || echo ldg)
  ADAPCC_ENGINE=$2 ncu --set full --clock-control none --import-source on -k regex:engine -s 4 -c 1 \
      -o $OUT/prof_${name}_$TAG python bench.py --mode $1 $SHORT > $OUT/ncu_${name}_$TAG.log 2>&1
done
for cfg in "16 1" "64 1" "16 0"; do
  set -- $cfg
  ncu --set full --clock-control none --import-source on -k regex:engine -s 3 -c 1 \
      -o $OUT/prof_acc${1}_red${2}_$TAG python scripts/debug/acc_one.py $1 $2 > $OUT/ncu_acc${1}_red${2}_$TAG.log 2>&1
done
python scripts/debug/host_overhead.py > $OUT/host_overhead_$TAG.log 2>&1
bash scripts/debug/host_floor.sh > $OUT/host_floor_$TAG.log 2>&1
ls -la $OUT
