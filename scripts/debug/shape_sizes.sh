#!/bin/bash
# TMA ring shape per message size on DIRECT plans (GPU box): the 1 CTA/SM x 3 x 64 KiB
# instantiation (ADAPCC_TMA_SHAPE=1) against 2 CTAs/SM x 3 x 32 KiB (=2), TMA engine forced,
# graph-timed, 1 MiB .. 256 MiB per rank, for AllReduce / AllGather / AlltoAll.
mkdir -p gpurun_out
for coll in allreduce allgather alltoall; do
  for sh in 1 2; do
    ADAPCC_TMA_SHAPE=$sh timeout 600 python scripts/sweep_sizes.py --coll $coll --graph --engine 1 \
      --min-log2 20 --max-log2 28 --out gpurun_out/shape_${coll}_s${sh}.json > /dev/null 2>&1
  done
done
python - <<'PY'
import json
for coll in ("allreduce", "allgather", "alltoall"):
    a = json.load(open(f"gpurun_out/shape_{coll}_s1.json")); b = json.load(open(f"gpurun_out/shape_{coll}_s2.json"))
    pa = a["points"] if isinstance(a, dict) else a; pb = b["points"] if isinstance(b, dict) else b
    for x, y in zip(pa, pb):
        print(coll, x.get("bytes_per_rank"), x.get("us"), y.get("us"))
PY
