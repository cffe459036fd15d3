import sys, time, ctypes, torch
sys.path.insert(0, '.')
import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import adapcc as A
from paper_conf_icdcs_zhaozw24_b200 import generator as G
n, cnt = 8, 1024
comm = pkg.Communicator.loopback(n, mode="direct")
comm.set_strategy("allreduce", G.allreduce_stars(n))
xs = [torch.randn(cnt, device="cuda") for _ in range(n)]
ys = [torch.empty_like(x) for x in xs]
L = A._load()
m = (1 << n) - 1
S, D = comm._arrays(xs, ys, m)
st = A._stream(None)
K = 5000
def bench(name, fn):
    for _ in range(100): fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(K): fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"{name:40s} {(t1-t0)/K*1e6:7.2f} us/call")
bench("python allreduce_lb", lambda: comm.allreduce_lb(xs, ys))
bench("ctypes adapcc_allreduce_lb (cached args)", lambda: L.adapcc_allreduce_lb(comm._h, S, D, cnt, 0, m, 0, st))
bench("_arrays", lambda: comm._arrays(xs, ys, m))
bench("_ready_mask", lambda: comm._ready_mask(None))
bench("_stream", lambda: A._stream(None))
bench("data_ptr x16", lambda: [t.data_ptr() for t in xs + ys])
bench("numel+dtype", lambda: (ys[0].numel(), A._dtype_code(ys[0])))
bench("empty kernel (torch add_)", lambda: xs[0].add_(0))
v = ctypes.c_uint64()
bench("ctypes trivial (launch_count)", lambda: L.adapcc_launch_count(comm._h, ctypes.byref(v)))
bench("ctypes allreduce_lb count=0", lambda: L.adapcc_allreduce_lb(comm._h, S, D, 0, 0, m, 0, st))
import torch
bench("raw stream", lambda: torch._C._cuda_getCurrentRawStream(0))
# device-limited? time with sync every 8 calls
def burst():
    for _ in range(8): L.adapcc_allreduce_lb(comm._h, S, D, cnt, 0, m, 0, st)
    torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(500): burst()
print("burst of 8 + sync per call", (time.perf_counter() - t0) / 4000 * 1e6)
# host-only enqueue cost: stream blocked by a long sleep kernel, 500 enqueues
for name, fn in [("ctypes allreduce_lb", lambda: L.adapcc_allreduce_lb(comm._h, S, D, cnt, 0, m, 0, st)),
                 ("python allreduce_lb", lambda: comm.allreduce_lb(xs, ys)),
                 ("torch add_", lambda: xs[0].add_(0))]:
    torch.cuda._sleep(int(2e9))
    t0 = time.perf_counter()
    for _ in range(500): fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"{name:40s} host-only {(t1-t0)/500*1e6:7.2f} us/call")
