"""ACCUMULATE AllReduce (phase 2: ready = {3, 6} of 8 virtual ranks, recv += sum) on the
TMA kernel across DIRECT ring shapes (stages x stage KiB x CTAs/SM), graph-timed.

    python scripts/debug/acc_variants.py --build   # here: compile the variants in-tree
    python scripts/debug/acc_variants.py           # GPU box: one subprocess per variant
"""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
VARIANTS = {"s3k64b1": (3, 64, 1), "s6k32b1": (6, 32, 1), "s4k48b1": (4, 48, 1),
            "s3k32b2": (3, 32, 2), "s2k96b1": (2, 96, 1), "s4k24b2": (4, 24, 2)}


def lib(v):
    return os.path.join(ROOT, "paper_conf_icdcs_zhaozw24_b200", f"libadapcc_acc_{v}.so")


def run_one():
    import torch
    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G
    n, R2 = 8, {3, 6}
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.config("engine", 1)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    out = {}
    for lg in (22, 24, 26, 28):
        count = (1 << lg) // 4
        xs = [torch.randn(count, device="cuda") for _ in range(n)]
        ys = [torch.randn(count, device="cuda") for _ in range(n)]
        fn = lambda: c.allreduce_lb([x if r in R2 else None for r, x in enumerate(xs)], ys, ready=R2, accumulate=True)  # noqa
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        reps = 10
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(reps):
                fn()
        t = []
        for _ in range(5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); g.replay(); b.record(); torch.cuda.synchronize()
            t.append(a.elapsed_time(b) / reps * 1e3)
        us = statistics.median(t)
        # traffic per call: 2 sources + 8 recv reads + 8 recv writes, S bytes each
        out[lg] = {"us": round(us, 2), "GBs_18S": round(18 * (1 << lg) / us / 1e3, 1)}
        del xs, ys
    print(json.dumps(out))


def main():
    if "--one" in sys.argv:
        return run_one()
    if "--build" in sys.argv:
        from paper_conf_icdcs_zhaozw24_b200 import _build
        for v, (s, k, b) in VARIANTS.items():
            _build.build(out=lib(v), defines=(f"ADAPCC_DIRECT_STAGES={s}", f"ADAPCC_DIRECT_STAGE_KB={k}",
                                              f"ADAPCC_DIRECT_MINB={b}"))
        return
    res = {}
    for v in VARIANTS:
        p = subprocess.run([sys.executable, __file__, "--one"], env=dict(os.environ, ADAPCC_LIB=lib(v)),
                           capture_output=True, text=True, timeout=300)
        line = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
        res[v] = json.loads(line[-1]) if line else {"error": p.stderr[-400:]}
        print(v, json.dumps(res[v]), flush=True)
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "acc_variants.json"), "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
