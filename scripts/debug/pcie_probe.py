"""Pinned host <-> device copy bandwidth on the box: one / two streams per direction, both directions."""
import json
import torch

N = 256 << 20
hs = [torch.empty(N, dtype=torch.uint8).pin_memory() for _ in range(4)]
ds = [torch.empty(N, dtype=torch.uint8, device="cuda") for _ in range(4)]
streams = [torch.cuda.Stream() for _ in range(4)]


def run(pairs, reps=4):
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for s in streams:
        s.wait_stream(torch.cuda.current_stream())
    for _ in range(reps):
        for k, (direction, si) in enumerate(pairs):
            with torch.cuda.stream(streams[si]):
                if direction == "h2d":
                    ds[k].copy_(hs[k], non_blocking=True)
                else:
                    hs[k].copy_(ds[k], non_blocking=True)
    for s in streams:
        torch.cuda.current_stream().wait_stream(s)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    return round(len(pairs) * reps * N / (ms * 1e-3) / 1e9, 1)


out = {"h2d_1stream": run([("h2d", 0)]), "h2d_2streams": run([("h2d", 0), ("h2d", 1)]),
       "d2h_1stream": run([("d2h", 0)]), "d2h_2streams": run([("d2h", 0), ("d2h", 1)]),
       "both_1+1": run([("h2d", 0), ("d2h", 1)]), "both_2+2": run([("h2d", 0), ("h2d", 1), ("d2h", 2), ("d2h", 3)])}
print(json.dumps(out))
