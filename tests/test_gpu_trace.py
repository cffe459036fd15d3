"""In-kernel trace (adapcc_config "trace", include/adapcc.h adapcc_trace_read):
every work item of a launch is executed exactly once, by one CTA, with
ordered timestamps, and the items' traffic adds up to the plan's -- for both
kernels and both LDG schedules.  Also checks that tracing does not change
results (bit-exact against the oracle)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from oracle import collectives as oc  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import generator as G  # noqa: E402
from synth import rank_tensors  # noqa: E402
from tests.gpu_util import bits, to_dev, to_host  # noqa: E402

pytestmark = pytest.mark.gpu
CTA = 0xFFFFFFFF


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


@pytest.mark.parametrize("engine,sched", [(0, 0), (0, 2), (1, 2)])
@pytest.mark.parametrize("mode", ["direct", "staged"])
def test_trace_items_exactly_once(engine, sched, mode):
    n, count = 4, (3 << 20) + 12
    text = G.allreduce_stars(n, chunk=1 << 20)
    comm = pkg.Communicator.loopback(n, device=0, scratch_bytes=256 << 20, mode=mode)
    comm.config("engine", engine)
    comm.config("sched", sched)
    comm.set_strategy("allreduce", text)
    xs = rank_tensors("f32", count, n, base=900)
    dx = [to_dev(x, "f32") for x in xs]
    dy = [torch.empty_like(t) for t in dx]
    comm.config("trace", 1 << 16)
    for _ in range(3):
        comm.allreduce_lb(dx, dy)
    recs, total = comm.trace()
    assert comm.get_async_error() == 0
    assert total == len(recs) > 0
    exp = oc.allreduce(xs, text, set(range(n)), "f32")
    for g in range(n):
        assert np.array_equal(bits(to_host(dy[g], "f32")), bits(exp[g]))
    st = pkg.plan_stats(text, count, "f32", (1 << n) - 1, mode=mode)
    launches = sorted(set(int(v) for v in recs["launch"]))
    assert len(launches) == 3
    for L in launches:
        r = recs[recs["launch"] == L]
        cta, it = r[r["item"] == CTA], r[r["item"] != CTA]
        assert len(set(int(c) for c in cta["cta"])) == len(cta)          # one record per CTA
        items = sorted(int(i) for i in it["item"])
        assert items == list(range(len(items)))                          # every item exactly once
        assert set(int(c) for c in it["cta"]) <= set(int(c) for c in cta["cta"])
        assert int(it["bytes"].sum()) == st["bytes_read"] + st["bytes_written"]
        for x in it:
            assert x["t0"] <= x["t1"] <= x["t2"]
        for c in cta:
            assert c["t0"] <= c["t1"] <= c["t2"]
            mine = it[it["cta"] == c["cta"]]
            if len(mine):
                assert c["t0"] <= mine["t0"].min() and mine["t2"].max() <= c["t2"]
    comm.config("trace", 0)
    with pytest.raises(pkg.AdapccError):
        comm.trace()
    comm.finalize()


def test_trace_capacity_drops_excess():
    n = 2
    comm = pkg.Communicator.loopback(n, device=0)
    comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=65536))
    comm.config("engine", 0)
    dx = [torch.randn(1 << 20, device="cuda") for _ in range(n)]
    dy = [torch.empty_like(t) for t in dx]
    comm.config("trace", 8)
    comm.allreduce_lb(dx, dy)
    recs, total = comm.trace()
    assert len(recs) == 8 and total > 8
    comm.allreduce_lb(dx, dy)       # the read emptied the buffer
    recs2, total2 = comm.trace()
    assert total2 == total and len(recs2) == 8
    comm.finalize()
