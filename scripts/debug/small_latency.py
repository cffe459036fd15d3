import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_icdcs_zhaozw24_b200 as pkg
from paper_conf_icdcs_zhaozw24_b200 import generator as G
n = 8
for cnt in (1024, 16384, 262144):
    comm = pkg.Communicator.loopback(n, mode="direct")
    comm.set_strategy("allreduce", G.allreduce_stars(n, chunk=262144))
    xs = [torch.randn(cnt, device="cuda") for _ in range(n)]
    ys = [torch.empty_like(x) for x in xs]
    for _ in range(50):
        comm.allreduce_lb(xs, ys)
    torch.cuda.synchronize()
    K = 2000
    t0 = time.perf_counter()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(K):
        comm.allreduce_lb(xs, ys)
    b.record()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print(f"count {cnt}: host enqueue {(t1-t0)/K*1e6:.2f} us/call, device {a.elapsed_time(b)/K*1e3:.2f} us/call, wall {(t2-t0)/K*1e6:.2f}")
    # graph
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        comm.allreduce_lb(xs, ys); torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            for _ in range(100):
                comm.allreduce_lb(xs, ys)
    torch.cuda.synchronize()
    a.record(); 
    for _ in range(20): g.replay()
    b.record(); torch.cuda.synchronize()
    print(f"   graph: {a.elapsed_time(b)/2000*1e3:.2f} us/call")
    comm.finalize()
