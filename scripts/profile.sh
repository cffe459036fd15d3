#!/bin/bash
# GPU-box profiling recipe (B200_PROFILING.md): bench line, launch list, and one
# ncu --set full capture of the engine kernel per (plan, engine) pair.
# Usage (under gpurun): bash scripts/profile.sh <tag>
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
cat $OUT/bench_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1 > /dev/null 2>&1
SHORT="--steps 3 --warmup 3 --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1"
for cfg in "direct 1" "direct 0" "staged 1" "staged 0"; do
  set -- $cfg
  name=${1}_$([ $2 = 1 ] && echo tma || echo ldg)
  ADAPCC_ENGINE=$2 ncu --set full --clock-control none --import-source on -k regex:engine -s 4 -c 1 \
      -o $OUT/prof_${name}_$TAG python bench.py --mode $1 $SHORT > $OUT/ncu_${name}_$TAG.log 2>&1
done
python bench.py --mode staged --steps 50 --warmup 5 --no-cpu-baseline --no-parity --no-sweep --e2e-steps 1 \
    > $OUT/bench_staged_$TAG.json 2>/dev/null
ls -la $OUT
