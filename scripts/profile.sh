#!/bin/bash
# GPU-box profiling recipe (B200_PROFILING.md): bench line, launch list, ncu --set full
# of the engine kernel for the DIRECT (bench) and STAGED (multi-process protocol) plans.
# Usage (under gpurun): bash scripts/profile.sh <tag>
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
cat $OUT/bench_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches_$TAG.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-parity --e2e-steps 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:engine_kernel -s 4 -c 1 \
    -o $OUT/prof_direct_$TAG python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-parity \
    --e2e-steps 1 > $OUT/ncu_direct_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:engine_kernel -s 4 -c 1 \
    -o $OUT/prof_staged_$TAG python bench.py --mode staged --steps 3 --warmup 3 --no-cpu-baseline \
    --no-parity --e2e-steps 1 > $OUT/ncu_staged_$TAG.log 2>&1
python bench.py --mode staged --steps 50 --warmup 5 --no-cpu-baseline --no-parity --e2e-steps 1 \
    > $OUT/bench_staged_$TAG.json 2>/dev/null
ls -la $OUT
