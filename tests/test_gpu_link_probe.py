"""adapcc_link_probe on the GPU (-m gpu): graph-captured probes give a
per-message alpha near the engine's launch floor (not host noise) and a
bandwidth below the copy peak; multi-process probes over CUDA IPC."""

import os
import socket
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import paper_conf_icdcs_zhaozw24_b200 as pkg  # noqa: E402
from paper_conf_icdcs_zhaozw24_b200 import costmodel as CM  # noqa: E402

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


@pytest.mark.parametrize("engine", ["sm", "ce"])
def test_loopback_profile(engine):
    comm = pkg.Communicator.loopback(3, scratch_bytes=256 << 20)
    p = CM.profile_links(comm, sizes=(1 << 16, 1 << 22), repeats=(1, 8), engine=engine)
    a, g = p["alpha_us"][0][1], p["beta_GBps"][0][1]
    # one GPU: a "link" is the HBM copy path (read + write of every byte)
    assert 0.3 < a < 15, p["alpha_us"]
    assert 300 < g < 8000, p["beta_GBps"]
    assert p["fanout"][0]["GBps_out"] > 0
    with pytest.raises(pkg.AdapccError):
        comm.link_probe({0}, 1 << 20, src=0)     # a rank cannot probe itself
    with pytest.raises(pkg.AdapccError):
        comm.link_probe({1}, 1000, src=0)        # not a multiple of 16
    comm.finalize()


def test_probe_messages_scale():
    """m messages take ~m times one message (the model t = m (alpha + beta s))."""
    comm = pkg.Communicator.loopback(2, scratch_bytes=256 << 20)
    t1 = comm.link_probe({1}, 1 << 22, messages=1, src=0, iters=40)
    t8 = comm.link_probe({1}, 1 << 22, messages=8, src=0, iters=10)
    assert 7.0 < t8 / t1 < 9.0, (t1, t8)
    comm.finalize()


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, n, port, q):
    try:
        sys.path.insert(0, ROOT)
        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=n)
        dev = rank % torch.cuda.device_count()
        torch.cuda.set_device(dev)
        comm = pkg.Communicator.init(scratch_bytes=64 << 20, device=dev)
        p = CM.profile_links(comm, sizes=(1 << 16, 1 << 20), repeats=(1, 4), engine="sm", iters=10)
        comm.finalize()
        dist.destroy_process_group()
        q.put((rank, True, p))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, False, traceback.format_exc() + repr(e)))


def test_multiprocess_probe_rounds():
    import torch.multiprocessing as mp
    n = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, n, port, q)) for r in range(n)]
    for p in ps:
        p.start()
    out = {}
    try:
        for _ in range(n):
            r, ok, p = q.get(timeout=300)
            out[r] = (ok, p)
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(n):
        assert out[r][0], out[r][1]
        p = out[r][1]
        for i in range(n):
            for j in range(n):
                if i != j:   # every link probed by its sender (one GPU here: time-sliced, so no bound on beta)
                    assert p["alpha_us"][i][j] is not None and f"{i}->{j}" in p["samples"]


def test_adapt_strategy_end_to_end():
    """Profile -> bandwidth-weighted stars -> cost-model chunk -> installed
    strategy; the next AllReduce runs on it bit-exactly (oracle replay of the
    new text)."""
    from oracle import collectives as oc
    from synth import rank_tensors
    from tests.gpu_util import bits, empty_dev, to_dev, to_host
    n, count = 4, 1_000_003
    comm = pkg.Communicator.loopback(n, scratch_bytes=256 << 20)
    text, prof, chunk = CM.adapt_strategy(comm, count * 4, ready={0, 1, 3}, sizes=(1 << 16, 1 << 20),
                                          repeats=(1, 4))
    assert chunk % 16 == 0 and "tree" in text
    xs = rank_tensors("f32", count, n)
    dy = [empty_dev(count, "f32") for _ in range(n)]
    comm.allreduce_lb([to_dev(x, "f32") for x in xs], dy, ready={0, 1, 3})
    torch.cuda.synchronize()
    exp = oc.allreduce(xs, text, {0, 1, 3}, "f32")
    assert all(np.array_equal(bits(to_host(y, "f32")), bits(e)) for y, e in zip(dy, exp))
    comm.finalize()
