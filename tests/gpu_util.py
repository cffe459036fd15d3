"""Helpers for GPU parity tests (numpy <-> torch; no method arithmetic)."""

import numpy as np

TORCH_DT = {"f32": "float32", "bf16": "bfloat16", "i32": "int32"}


def to_dev(a, dtype):
    import torch
    t = torch.from_numpy(np.ascontiguousarray(a))
    if dtype == "bf16":
        t = t.view(torch.int16).cuda().view(torch.bfloat16)   # bit patterns preserved
    else:
        t = t.cuda()
    return t


def to_host(t, dtype):
    import torch
    if dtype == "bf16":
        return t.view(torch.int16).cpu().numpy().view(np.uint16)
    return t.cpu().numpy()


def bits(a):
    a = np.asarray(a)
    return a.view(np.uint16) if a.dtype == np.uint16 else a.view(np.uint32)


def empty_dev(n_elems, dtype, fill_bits=0x5A):
    import torch
    dt = getattr(torch, TORCH_DT[dtype])
    t = torch.empty(n_elems, dtype=dt, device="cuda")
    t.view(torch.uint8).fill_(fill_bits)
    return t
