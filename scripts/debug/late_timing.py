"""Late-join phase timings in loopback (DIRECT, 8 virtual ranks, stragglers {3, 6}):
(a) phase 1 when both stragglers signalled before it (every piece folds them),
(b) the complement after (a) (nothing left to add), (c) phase 1 with no signal,
(d) the complement after (c) (adds both to every piece), vs a plain full AllReduce."""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402

n, R1, R2 = 8, {0, 1, 2, 4, 5, 7}, [3, 6]
out = {}
for mib in (25, 100):
    count = (mib << 20) // 4
    c = pkg.Communicator.loopback(n, mode="direct", scratch_bytes=64 << 20)
    c.set_strategy("allreduce", G.allreduce_stars(n))
    dx = [torch.randn(count, device="cuda") for _ in range(n)]
    dy = [torch.empty_like(x) for x in dx]

    def t(fn, reps=5):
        best = 1e9
        for _ in range(reps):
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); fn(); b.record(); torch.cuda.synchronize()
            best = min(best, a.elapsed_time(b))
        return round(best, 4)

    for _ in range(3):
        c.allreduce_lb(dx, dy)
        c.allreduce_lb(dx, dy, ready=R1, late="join")
        c.allreduce_lb(dx, dy, ready=R1, late="complement")
    torch.cuda.synchronize()
    row = {"full": t(lambda: c.allreduce_lb(dx, dy))}
    res = {}
    for case in ("all", "none"):
        pa, pb = [], []
        for _ in range(5):
            tk = c.late_ticket() + 1
            if case == "all":
                for r in R2:
                    c.signal_ready(rank=r, ticket=tk)
            torch.cuda.synchronize()
            a, b, e = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            a.record(); c.allreduce_lb(dx, dy, ready=R1, late="join"); b.record()
            c.allreduce_lb(dx, dy, ready=R1, late="complement"); e.record()
            torch.cuda.synchronize()
            pa.append(a.elapsed_time(b)); pb.append(b.elapsed_time(e))
        res[case] = (round(min(pa), 4), round(min(pb), 4))
    row["join_signalled_before"], row["complement_after_that"] = res["all"]
    row["join_no_signal"], row["complement_all_missing"] = res["none"]
    row["plain_partial_phase1"] = t(lambda: c.allreduce_lb([x if r in R1 else None for r, x in enumerate(dx)], dy, ready=R1))
    out[mib] = row
    c.finalize()
print(json.dumps(out))
