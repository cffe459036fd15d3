"""Link profiler host logic (NEXT-2) on CPU: a synthetic link model
stands in for adapcc_link_probe; the profiler must recover alpha / beta per
link, use permutation rounds (Fig. 5(b)), and assemble the matrix across ranks
(world size 2 over gloo)."""

import os
import socket

import pytest

from paper_conf_icdcs_zhaozw24_b200 import costmodel as CM


class FakeComm:
    """t(messages, bytes) = messages * (alpha_ij + beta_ij * bytes): the
    paper's model of a link, per (src, dst); records the probe calls."""

    def __init__(self, n, rank, loopback, alpha, beta):
        self.nranks, self.rank, self.loopback = n, rank, loopback
        self.alpha, self.beta = alpha, beta
        self.calls = []

    def link_probe(self, dst, nbytes, messages=1, engine="sm", iters=20, src=-1):
        s = self.rank if src < 0 else src
        self.calls.append((s, tuple(sorted(dst)), nbytes, messages))
        if not dst:
            return 0.0
        return max(messages * (self.alpha[s][d] + self.beta[s][d] * nbytes) for d in dst)


def _links(n):
    alpha = [[2e-6 + 1e-7 * (i + 2 * j) for j in range(n)] for i in range(n)]
    beta = [[1.0 / ((600 + 10 * i + j) * 1e9) for j in range(n)] for i in range(n)]
    return alpha, beta


def test_loopback_recovers_alpha_beta():
    n = 4
    alpha, beta = _links(n)
    p = CM.profile_links(FakeComm(n, 0, True, alpha, beta))
    for j in range(1, n):
        assert p["alpha_us"][0][j] == pytest.approx(alpha[0][j] * 1e6, rel=1e-6)
        assert p["beta_GBps"][0][j] == pytest.approx(1 / beta[0][j] / 1e9, rel=1e-6)
    f = p["fanout"][0]
    assert f["dsts"] == n - 1 and f["GBps_per_dst"] > 0
    a, b = CM.links_to_model(p)
    assert a[0][1] == pytest.approx(alpha[0][1]) and a[2][3] > 0 and b[3][2] > 0   # unmeasured: mean fill


def test_probe_calls_follow_the_paper_shapes():
    """For every (s, m): m messages of s, then one message of m*s."""
    n = 3
    alpha, beta = _links(n)
    c = FakeComm(n, 0, True, alpha, beta)
    CM.profile_links(c, sizes=(4096, 65536), repeats=(1, 8))
    to1 = [x for x in c.calls if x[1] == (1,)]
    assert [(b, m) for _, _, b, m in to1] == [(4096, 1), (4096, 1), (4096, 8), (32768, 1),
                                               (65536, 1), (65536, 1), (65536, 8), (524288, 1)]


def test_per_gpu_bandwidth_and_chunk():
    n = 4
    alpha, beta = _links(n)
    p = CM.profile_links(FakeComm(n, 0, True, alpha, beta))
    bw = CM.per_gpu_bandwidth(p)
    assert len(bw) == n and bw[0] == pytest.approx(min(1 / beta[0][j] / 1e9 for j in range(1, n)), rel=1e-6)
    best, scored = CM.chunk_from_profile(p, 256 << 20)
    assert best in [c for _, c in scored]
    assert min(t for t, _ in scored) == pytest.approx(dict((c, t) for t, c in scored)[best])


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, q):
    import torch.distributed as dist
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        alpha, beta = _links(n)
        c = FakeComm(n, rank, False, alpha, beta)
        p = CM.profile_links(c, sizes=(1 << 16, 1 << 20), repeats=(1, 4))
        # every rank made the same number of (collective) probe calls
        ncalls = [None] * n
        dist.all_gather_object(ncalls, len(c.calls))
        dist.destroy_process_group()
        q.put((rank, p, ncalls, c.calls))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc() + repr(e), None, None))


@pytest.mark.parametrize("n", [2, 3])
def test_multiprocess_rounds_gloo(n):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    out = {}
    for _ in range(n):
        r, p, ncalls, calls = q.get(timeout=120)
        assert isinstance(p, dict), p
        out[r] = (p, ncalls, calls)
    for p in ps:
        p.join(timeout=30)
    alpha, beta = _links(n)
    for r, (p, ncalls, calls) in out.items():
        assert len(set(ncalls)) == 1
        for i in range(n):
            for j in range(n):
                if i != j:   # every link measured by its sender, gathered everywhere
                    assert p["alpha_us"][i][j] == pytest.approx(alpha[i][j] * 1e6, rel=1e-6)
        # rank r probes (r + i) % n in round i: one partner per round, a permutation overall
        partners = [c[1] for c in calls if c[1] and len(c[1]) == 1]
        assert sorted({x[0] for x in partners}) == sorted({(r + i) % n for i in range(1, n)})


class FakeStrategyComm(FakeComm):
    def __init__(self, *a, **k):
        super().__init__(*a, **k)
        self.set_calls, self.config_calls = [], []

    def set_strategy(self, coll, text):
        self.set_calls.append((coll, text))

    def config(self, key, value):
        self.config_calls.append((key, value))


def test_adapt_strategy_weights_follow_bandwidth():
    """A GPU with half the link bandwidth roots a smaller partition; the
    chunk is the cost model's choice; the strategy is installed."""
    from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
    n = 4
    alpha = [[2e-6] * n for _ in range(n)]
    beta = [[1.0 / (800e9 if i != 2 else 400e9)] * n for i in range(n)]
    c = FakeStrategyComm(n, 0, True, alpha, beta)
    # loopback probes only rank 0's links: give every rank its own row
    prof = CM.profile_links(c)
    for i in range(n):
        for j in range(n):
            if i != j:
                prof["beta_GBps"][i][j] = 1.0 / beta[i][j] / 1e9
    text, _, chunk = CM.adapt_strategy(c, 64 << 20, profile=prof)
    assert c.set_calls == [("allreduce", text)] and ("default_chunk", chunk) in c.config_calls
    w = [A.strategy_sub(text, m)[0] for m in range(n)]
    assert w[2] < min(w[g] for g in range(n) if g != 2)
    assert chunk == CM.chunk_from_profile(prof, 64 << 20, text_for_chunk=lambda ch: text.replace(
        f"chunk={chunk}", f"chunk={ch}"))[0]
