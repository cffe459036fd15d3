"""Tuning sweep (GPU box): engine variants x chunk sizes through bench.py.

    python scripts/sweep_engine.py --build      # here: compile variants in-tree
    python scripts/sweep_engine.py              # on the GPU: run, write gpurun_out/sweep.json
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
VARIANTS = {  # TMA pipeline shapes: stages x stage KiB x CTAs/SM
    "s3k32b2": ("ADAPCC_TMA_STAGES=3", "ADAPCC_TMA_STAGE_KB=32", "ADAPCC_TMA_MINB=2"),
    "s4k32b1": ("ADAPCC_TMA_STAGES=4", "ADAPCC_TMA_STAGE_KB=32", "ADAPCC_TMA_MINB=1"),
    "s6k32b1": ("ADAPCC_TMA_STAGES=6", "ADAPCC_TMA_STAGE_KB=32", "ADAPCC_TMA_MINB=1"),
    "s5k40b1": ("ADAPCC_TMA_STAGES=5", "ADAPCC_TMA_STAGE_KB=40", "ADAPCC_TMA_MINB=1"),
    "s4k48b1": ("ADAPCC_TMA_STAGES=4", "ADAPCC_TMA_STAGE_KB=48", "ADAPCC_TMA_MINB=1"),
    "s3k64b1": ("ADAPCC_TMA_STAGES=3", "ADAPCC_TMA_STAGE_KB=64", "ADAPCC_TMA_MINB=1"),
}


def lib(v):
    return os.path.join(ROOT, "paper_conf_icdcs_zhaozw24_b200", f"libadapcc_{v}.so")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--build", action="store_true")
    ap.add_argument("--variants", default=",".join(VARIANTS))
    ap.add_argument("--chunks", default="256")
    ap.add_argument("--extra", default="")
    ap.add_argument("--pieces", default="0", help="ADAPCC_PIECE_KIB values (0 = auto)")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.json"))
    a = ap.parse_args()
    if a.build:
        from paper_conf_icdcs_zhaozw24_b200 import _build
        for v in a.variants.split(","):
            _build.build(out=lib(v), defines=VARIANTS[v])
        return
    res = []
    for v in a.variants.split(","):
        for c, pk in [(c, pk) for c in a.chunks.split(",") for pk in a.pieces.split(",")]:
            env = dict(os.environ, ADAPCC_LIB=lib(v), ADAPCC_PIECE_KIB=pk)
            cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "50", "--warmup", "5",
                   "--no-cpu-baseline", "--no-parity", "--e2e-steps", "1", "--chunk-kib", c] + a.extra.split()
            p = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=600)
            line = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
            if not line:
                res.append({"variant": v, "chunk_kib": int(c), "error": p.stderr[-500:]})
                continue
            d = json.loads(line[-1])
            res.append({"variant": v, "chunk_kib": int(c), "piece_kib": int(pk), "busbw": d["value"],
                        "frac": d["roofline"]["frac"], "kernel_ms": d["roofline"]["kernel_ms"],
                        "clocks": d["clocks"]})
            print(json.dumps(res[-1]), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
