"""In-kernel trace of engine launches (adapcc_config "trace"): where a call's
time goes, per CTA and per work item, plus a Chrome-trace timeline
(chrome://tracing / Perfetto) -- the timeline view nsys would give, which this
image does not have.

    python scripts/trace_report.py [--coll allreduce] [--bytes-per-rank 8388608]
        [--ranks 8] [--engine 2] [--calls 20] [--out gpurun_out/trace]

Runs `calls` back-to-back loopback calls with tracing on, then reports for the
median launch: kernel span (first CTA entry -> last CTA exit), entry spread,
per-CTA busy fraction, the idle tail (last exit - median exit), item count,
item time and inputs-wait percentiles, and per-item bandwidth.  Writes
<out>.json (the summary) and <out>_timeline.json (the median launch as Chrome
trace events: one row per CTA, one slice per item)."""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def pct(v, q):
    v = sorted(v)
    return v[min(len(v) - 1, int(q * (len(v) - 1) + 0.5))] if v else 0


def summarize(recs, launch):
    import numpy as np
    r = recs[recs["launch"] == launch]
    cta = r[r["item"] == 0xFFFFFFFF]
    it = r[r["item"] != 0xFFFFFFFF]
    t_start, t_end = int(cta["t0"].min()), int(cta["t2"].max())
    span = (t_end - t_start) / 1e3
    exits = sorted(int(x) for x in cta["t2"])
    busy = {}
    for x in it:
        busy[int(x["cta"])] = busy.get(int(x["cta"]), 0) + int(x["t2"] - x["t0"])
    dur = [(int(x["t2"]) - int(x["t0"])) / 1e3 for x in it]
    wait = [(int(x["t1"]) - int(x["t0"])) / 1e3 for x in it]
    bw = [int(x["bytes"]) / max(1, int(x["t2"]) - int(x["t0"])) for x in it]  # GB/s
    return {
        "launch": int(launch), "ctas": int(len(cta)), "items": int(len(it)),
        "bytes": int(it["bytes"].sum()),
        "span_us": round(span, 3),
        "entry_spread_us": round((int(cta["t0"].max()) - t_start) / 1e3, 3),
        "ready_after_entry_us_p50": round(pct([(int(c["t1"]) - int(c["t0"])) / 1e3 for c in cta], 0.5), 3),
        "first_item_start_us": round(pct([(int(x["t0"]) - t_start) / 1e3 for x in it], 0.0), 3),
        "tail_us": round((exits[-1] - exits[len(exits) // 2]) / 1e3, 3),
        "busy_frac_mean": round(statistics.mean(busy.values()) / max(1, t_end - t_start), 3) if busy else 0,
        "item_us": {"p10": round(pct(dur, .1), 3), "p50": round(pct(dur, .5), 3), "p90": round(pct(dur, .9), 3),
                    "max": round(max(dur), 3) if dur else 0},
        "wait_us": {"p50": round(pct(wait, .5), 3), "p90": round(pct(wait, .9), 3),
                    "max": round(max(wait), 3) if wait else 0},
        "item_gbs": {"p10": round(pct(bw, .1), 1), "p50": round(pct(bw, .5), 1), "p90": round(pct(bw, .9), 1)},
        "items_per_cta_max": int(max(np.bincount(it["cta"].astype(np.int64)))) if len(it) else 0,
        "algbw_span_gbs": round(int(it["bytes"].sum()) / max(1, t_end - t_start), 1),
    }


def timeline(recs, launch):
    r = recs[recs["launch"] == launch]
    t_start = int(r[r["item"] == 0xFFFFFFFF]["t0"].min())
    ev = []
    for x in r:
        c = int(x["cta"])
        if int(x["item"]) == 0xFFFFFFFF:
            ev.append({"name": "cta", "ph": "X", "pid": 0, "tid": c, "ts": (int(x["t0"]) - t_start) / 1e3,
                       "dur": (int(x["t2"]) - int(x["t0"])) / 1e3, "args": {"ready_us": (int(x["t1"]) - int(x["t0"])) / 1e3}})
        else:
            ev.append({"name": f"item {int(x['item'])}", "ph": "X", "pid": 1, "tid": c,
                       "ts": (int(x["t0"]) - t_start) / 1e3, "dur": (int(x["t2"]) - int(x["t0"])) / 1e3,
                       "args": {"wait_us": (int(x["t1"]) - int(x["t0"])) / 1e3, "bytes": int(x["bytes"])}})
    return {"traceEvents": ev, "displayTimeUnit": "ns"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--coll", default="allreduce", choices=["allreduce", "allgather", "alltoall"])
    ap.add_argument("--bytes-per-rank", type=int, default=8 << 20)
    ap.add_argument("--ranks", type=int, default=8)
    ap.add_argument("--mode", default="direct")
    ap.add_argument("--engine", type=int, default=2)
    ap.add_argument("--calls", type=int, default=20)
    ap.add_argument("--accumulate-ready", default=None,
                    help="allreduce as phase 2: comma-separated ready ranks, recv += sum (ACCUMULATE)")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "trace"))
    ap.add_argument("--raw", action="store_true", help="also save every record (<out>_raw.npy)")
    a = ap.parse_args()
    import torch

    import paper_conf_icdcs_zhaozw24_b200 as pkg
    from paper_conf_icdcs_zhaozw24_b200 import generator as G

    n = a.ranks
    comm = pkg.Communicator.loopback(n, scratch_bytes=1 << 30, mode=a.mode)
    comm.config("engine", a.engine)
    text = {"allreduce": G.allreduce_stars(n), "allgather": G.allgather_stars(n),
            "alltoall": G.alltoall_direct(n)}[a.coll]
    comm.set_strategy(a.coll, text)
    count = a.bytes_per_rank // 4
    if a.coll == "allgather":
        xs = [torch.randn(count // n, device="cuda") for _ in range(n)]
        ys = [torch.empty(count // n * n, device="cuda") for _ in range(n)]
    else:
        xs = [torch.randn(count, device="cuda") for _ in range(n)]
        ys = [torch.empty_like(x) for x in xs]
    fn = getattr(comm, a.coll + "_lb")
    if a.accumulate_ready:
        R = {int(r) for r in a.accumulate_ready.split(",")}
        xs = [x if r in R else None for r, x in enumerate(xs)]
        fn = lambda x_, y_: comm.allreduce_lb(x_, y_, ready=R, accumulate=True)  # noqa: E731
    for _ in range(3):
        fn(xs, ys)
    torch.cuda.synchronize()
    comm.config("trace", 1 << 22)
    l0 = comm.launch_count()
    for _ in range(a.calls):
        fn(xs, ys)
    recs, total = comm.trace()
    assert comm.get_async_error() == 0
    launches = sorted(set(int(v) for v in recs["launch"]))
    sums = [summarize(recs, L) for L in launches]
    med = sorted(sums, key=lambda s: s["span_us"])[len(sums) // 2]
    out = {"coll": a.coll, "ranks": n, "bytes_per_rank": a.bytes_per_rank, "mode": a.mode,
           "engine": comm.last_engine(), "calls": a.calls, "first_launch": l0, "records": int(total),
           "median_launch": med,
           "span_us_all": [s["span_us"] for s in sums]}
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    json.dump(out, open(a.out + ".json", "w"), indent=1)
    json.dump(timeline(recs, med["launch"]), open(a.out + "_timeline.json", "w"))
    if a.raw:
        import numpy as np
        np.save(a.out + "_raw.npy", recs)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
