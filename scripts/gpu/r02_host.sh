mkdir -p gpurun_out
python - > gpurun_out/host_prepared.log 2>&1 <<'PY'
import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import generator as G
n = 8
for cnt in (256, 4096, 65536):
    comm = pkg.Communicator.loopback(n, mode="direct")
    comm.set_strategy("allreduce", G.allreduce_stars(n))
    xs = [torch.randn(cnt, device="cuda") for _ in range(n)]
    ys = [torch.empty_like(x) for x in xs]
    call = comm.prepare_allreduce_lb(xs, ys)
    for name, fn in (("prepared", call), ("api", lambda: comm.allreduce_lb(xs, ys))):
        for _ in range(200): fn()
        torch.cuda.synchronize()
        K = 2000
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter(); a.record()
        for _ in range(K): fn()
        b.record(); torch.cuda.synchronize(); t1 = time.perf_counter()
        torch.cuda._sleep(int(2e8))
        h0 = time.perf_counter()
        for _ in range(300): fn()
        h1 = time.perf_counter(); torch.cuda.synchronize()
        print(f"{cnt*4:7d} B/rank {name:9s} back-to-back {a.elapsed_time(b)*1e3/K:6.2f} us/call (events) "
              f"{(t1-t0)/K*1e6:6.2f} (wall)   host-only {(h1-h0)/300*1e6:6.2f} us/call")
    comm.finalize()
PY

