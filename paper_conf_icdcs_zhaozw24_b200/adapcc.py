"""Thin Python binding of libadapcc.so (include/adapcc.h): argument marshalling only.

Every step of the collective runs in the CUDA engine behind the C ABI; there
is no Python or CPU fallback -- if the library is missing or a call fails,
this module raises.  torch is used only for tensors, the current stream and
the process group used to bootstrap IPC handles (the paper's set-up
AllGather), as the north star requires.

API (mirrors the paper's ``adapcc.init()/setup()/allreduce()``):
    comm = Communicator.init(group)                 # one process per GPU
    comm = Communicator.loopback(n, mode="direct")  # n virtual ranks, 1 GPU
    comm.set_strategy("allreduce", text)
    comm.allreduce(x, out, ready={...}, accumulate=False)
    comm.allgather(x, out, ready) ; comm.alltoall(x, out, ready)
    comm.allreduce_lb([x_r], [y_r], ready, accumulate)  # loopback
Host-only helpers (no GPU): strategy_check, strategy_tuples, strategy_sub,
strategy_partition, plan_stats.
"""

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
# ADAPCC_LIB selects an alternative in-tree build (tuning sweeps only)
_LIB_PATH = os.environ.get("ADAPCC_LIB") or os.path.join(_PKG, "libadapcc.so")

SUCCESS, INVALID_ARGUMENT, INVALID_STRATEGY, UNSUPPORTED, CUDA, BOOTSTRAP, OOM, TIMEOUT, MISMATCH = range(9)
COLL = {"allreduce": 0, "allgather": 1, "alltoall": 2, "reduce": 3, "broadcast": 4,
        "reducescatter": 5}
MODE = {"direct": 0, "staged": 1}
FLAG_ACCUMULATE = 0x1
FLAG_LATE_JOIN = 0x2
FLAG_LATE_COMPLEMENT = 0x4
DTYPE_CODE = {"f32": 0, "bf16": 1, "i32": 2}

_lib = None


class AdapccError(RuntimeError):
    def __init__(self, code, where=""):
        self.code = code
        msg = _load().adapcc_strerror(code).decode() if code >= 0 else "error"
        if code == CUDA:
            msg += ": " + _load().adapcc_last_cuda_error().decode()
        super().__init__(f"{where}: adapcc error {code} ({msg})")


class PlanStats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_uint64) for k in (
        "tasks", "items", "levels", "segments", "bytes_read", "bytes_written",
        "remote_bytes", "arena_bytes")]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


AG_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t,
                         ctypes.c_void_p)


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} is missing: build it with "
                          "`python -m paper_conf_icdcs_zhaozw24_b200._build` (there is no fallback)")
    L = ctypes.CDLL(_LIB_PATH)
    vp, sz, u64, i32, i64 = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint64, ctypes.c_int, ctypes.c_int64
    pp = ctypes.POINTER(ctypes.c_void_p)
    sig = {
        "adapcc_init": [ctypes.POINTER(vp), i32, i32, i32, sz, AG_FN, vp],
        "adapcc_init_loopback": [ctypes.POINTER(vp), i32, i32, sz, i32],
        "adapcc_set_strategy": [vp, i32, ctypes.c_char_p, vp],
        "adapcc_allreduce": [vp, vp, vp, sz, i32, u64, ctypes.c_uint, vp],
        "adapcc_allgather": [vp, vp, vp, sz, i32, u64, vp],
        "adapcc_alltoall": [vp, vp, vp, sz, i32, u64, vp],
        "adapcc_allreduce_lb": [vp, pp, pp, sz, i32, u64, ctypes.c_uint, vp],
        "adapcc_allgather_lb": [vp, pp, pp, sz, i32, u64, vp],
        "adapcc_alltoall_lb": [vp, pp, pp, sz, i32, u64, vp],
        "adapcc_reduce": [vp, vp, vp, sz, i32, i32, u64, ctypes.c_uint, vp],
        "adapcc_broadcast": [vp, vp, vp, sz, i32, i32, u64, vp],
        "adapcc_reducescatter": [vp, vp, vp, sz, i32, u64, ctypes.c_uint, vp],
        "adapcc_reduce_lb": [vp, pp, pp, sz, i32, i32, u64, ctypes.c_uint, vp],
        "adapcc_broadcast_lb": [vp, pp, pp, sz, i32, i32, u64, vp],
        "adapcc_reducescatter_lb": [vp, pp, pp, sz, i32, u64, ctypes.c_uint, vp],
        "adapcc_register_buffer": [vp, vp, sz, ctypes.POINTER(i32)],
        "adapcc_deregister_buffer": [vp, i32],
        "adapcc_collective_zc": [vp, i32, i32, sz, i32, sz, sz, i32, i32, u64, ctypes.c_uint, vp],
        "adapcc_alltoallv": [vp, vp, vp, ctypes.POINTER(u64), i32, u64, vp],
        "adapcc_alltoallv_lb": [vp, pp, pp, ctypes.POINTER(u64), i32, u64, vp],
        "adapcc_late_ticket": [vp, ctypes.POINTER(u64)],
        "adapcc_nvls_setup": [vp, sz, ctypes.c_char_p, sz],
        "adapcc_late_advance": [vp, ctypes.POINTER(u64)],
        "adapcc_link_probe": [vp, i32, u64, sz, i32, i32, i32, ctypes.POINTER(ctypes.c_double)],
        "adapcc_signal_ready": [vp, i32, u64, vp],
        "adapcc_ready_board": [vp, ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(i32)],
        "adapcc_spin": [vp, u64, vp],
        "adapcc_coord_decide": [vp, i32, u64, u64, ctypes.POINTER(ctypes.c_double), ctypes.c_double,
                                ctypes.c_double, ctypes.POINTER(u64), ctypes.POINTER(i32),
                                ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)],
        "adapcc_coord_await": [vp, i32, u64, u64, vp, ctypes.c_double, ctypes.c_double, ctypes.c_double,
                               ctypes.POINTER(u64)],
        "adapcc_get_async_error": [vp],
        "adapcc_finalize": [vp],
        "adapcc_config": [vp, ctypes.c_char_p, i64],
        "adapcc_launch_count": [vp, ctypes.POINTER(u64)],
        "adapcc_last_engine": [vp, ctypes.POINTER(i32)],
        "adapcc_trace_read": [vp, vp, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32),
                              ctypes.POINTER(ctypes.c_uint32)],
        "adapcc_exclude": [vp, u64, AG_FN, vp],
        "adapcc_members": [vp, ctypes.POINTER(u64)],
        "adapcc_strategy_check": [ctypes.c_char_p, ctypes.POINTER(i32), ctypes.POINTER(i32),
                                  ctypes.POINTER(i32), ctypes.c_char_p, sz],
        "adapcc_strategy_tuples": [ctypes.c_char_p, i32, u64, ctypes.POINTER(ctypes.c_uint8),
                                   ctypes.POINTER(ctypes.c_int32)],
        "adapcc_strategy_sub": [ctypes.c_char_p, i32, ctypes.POINTER(i64), ctypes.POINTER(i64),
                                ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int32)],
        "adapcc_strategy_route": [ctypes.c_char_p, i32, i32, i32, ctypes.POINTER(ctypes.c_int32),
                                  ctypes.POINTER(i32)],
        "adapcc_strategy_partition": [ctypes.c_char_p, u64, i32, i32, ctypes.POINTER(u64),
                                      ctypes.POINTER(i32)],
        "adapcc_plan_stats": [ctypes.c_char_p, u64, i32, u64, ctypes.c_uint, i32, i32, sz, u64,
                              ctypes.POINTER(PlanStats)],
        "adapcc_plan_items": [ctypes.c_char_p, u64, i32, u64, ctypes.c_uint, i32, i32, sz, i32, i32,
                              ctypes.c_uint32, i32, i32, vp, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32),
                              vp, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32)],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    L.adapcc_strerror.argtypes = [ctypes.c_int]
    L.adapcc_strerror.restype = ctypes.c_char_p
    L.adapcc_last_cuda_error.argtypes = []
    L.adapcc_last_cuda_error.restype = ctypes.c_char_p
    _lib = L
    return L


def lib_path():
    return _LIB_PATH


def _check(code, where):
    if code != SUCCESS:
        raise AdapccError(code, where)


def _mask(ready, n):
    if ready is None:
        return (1 << n) - 1
    if isinstance(ready, int):
        return ready
    m = 0
    for r in ready:
        m |= 1 << int(r)
    return m


_TORCH_CODES = None


def _dtype_code(t):
    global _TORCH_CODES
    if _TORCH_CODES is None:
        import torch
        _TORCH_CODES = {torch.float32: 0, torch.bfloat16: 1, torch.int32: 2}
    code = _TORCH_CODES.get(t.dtype)
    if code is None:
        raise TypeError(f"unsupported dtype {t.dtype}")
    return code


def _stream(stream, device=None):
    """Raw cudaStream_t: the given torch stream, else the current stream of
    `device` (default: the current device)."""
    import torch
    if stream is not None:
        return ctypes.c_void_p(stream.cuda_stream)
    dev = torch.cuda.current_device() if device is None else device
    return ctypes.c_void_p(torch._C._cuda_getCurrentRawStream(dev))


def _late_flag(late):
    return {None: 0, "join": FLAG_LATE_JOIN, "complement": FLAG_LATE_COMPLEMENT}[late]


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else ctypes.c_void_p(0)


# ------------------------------------------------------------ host-only helpers
def strategy_check(text):
    L = _load()
    n, c, m = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    err = ctypes.create_string_buffer(256)
    code = L.adapcc_strategy_check(text.encode(), ctypes.byref(n), ctypes.byref(c),
                                   ctypes.byref(m), err, 256)
    if code != SUCCESS:
        raise AdapccError(code, "strategy_check: " + err.value.decode())
    return n.value, c.value, m.value


def strategy_tuples(text, sub, mask):
    L = _load()
    n, _, _ = strategy_check(text)
    tup = (ctypes.c_uint8 * (4 * n))()
    nfl = (ctypes.c_int32 * n)()
    _check(L.adapcc_strategy_tuples(text.encode(), sub, mask, tup, nfl), "strategy_tuples")
    return [tuple(bool(tup[4 * g + i]) for i in range(4)) for g in range(n)], list(nfl)


def strategy_sub(text, sub):
    L = _load()
    n, _, _ = strategy_check(text)
    w, c = ctypes.c_int64(), ctypes.c_int64()
    par = (ctypes.c_int32 * n)()
    src = ctypes.c_int32()
    _check(L.adapcc_strategy_sub(text.encode(), sub, ctypes.byref(w), ctypes.byref(c), par,
                                 ctypes.byref(src)), "strategy_sub")
    return w.value, c.value, list(par), src.value


def strategy_route(text, sub, src, dst):
    """Relay ranks of AlltoAll flow src -> dst in a2a line `sub` ([] = direct)."""
    L = _load()
    n, _, _ = strategy_check(text)
    hops = (ctypes.c_int32 * n)()
    nh = ctypes.c_int()
    _check(L.adapcc_strategy_route(text.encode(), sub, src, dst, hops, ctypes.byref(nh)),
           "strategy_route")
    return list(hops[:nh.value])


def strategy_partition(text, count, dtype, src=-1):
    L = _load()
    _, _, m = strategy_check(text)
    b = (ctypes.c_uint64 * (m + 1))()
    nb = ctypes.c_int()
    _check(L.adapcc_strategy_partition(text.encode(), count, DTYPE_CODE[dtype], src, b,
                                       ctypes.byref(nb)), "strategy_partition")
    return list(b[:nb.value])


def plan_stats(text, count, dtype, mask, accumulate=False, mode="direct", rank=-1, scratch_bytes=0,
               members=None):
    """Byte/task accounting of a call's plan; members: live ranks (None = all)."""
    L = _load()
    st = PlanStats()
    mm = 0 if members is None else sum(1 << g for g in members)
    _check(L.adapcc_plan_stats(text.encode(), count, DTYPE_CODE[dtype], mask,
                               FLAG_ACCUMULATE if accumulate else 0, MODE[mode], rank,
                               scratch_bytes, mm, ctypes.byref(st)), "plan_stats")
    return st.as_dict()


def plan_items(text, count, dtype, mask, grid, tma=False, accumulate=False, mode="direct", rank=-1,
               scratch_bytes=0, piece_kib=0, taper=0, segment=0, late=None):
    """Work items (claim order) and tasks of one segment of a call's plan, as
    numpy structured arrays (include/adapcc.h adapcc_plan_items)."""
    import numpy as np
    L = _load()
    idt = np.dtype([("task", "<u4"), ("chunk", "<u4"), ("off", "<u4"), ("len", "<u4")])
    tdt = np.dtype([("lo", "<u8"), ("hi", "<u8"), ("chunk_elems", "<u4"), ("nchunks", "<u4"),
                    ("nsrc", "<u2"), ("ndst", "<u2"), ("nwait", "<u2"), ("npost", "<u2"),
                    ("level", "<u4"), ("owner", "<u4")])
    ni, nt = ctypes.c_uint32(), ctypes.c_uint32()
    flags = (FLAG_ACCUMULATE if accumulate else 0) | _late_flag(late)
    args = (text.encode(), count, DTYPE_CODE[dtype], mask, flags, MODE[mode],
            rank, scratch_bytes, grid, 1 if tma else 0, piece_kib, taper, segment)
    _check(L.adapcc_plan_items(*args, None, 0, ctypes.byref(ni), None, 0, ctypes.byref(nt)), "plan_items")
    items, tasks = np.zeros(ni.value, dtype=idt), np.zeros(nt.value, dtype=tdt)
    _check(L.adapcc_plan_items(*args, items.ctypes.data, ni.value, ctypes.byref(ni), tasks.ctypes.data,
                               nt.value, ctypes.byref(nt)), "plan_items")
    return items, tasks


# --------------------------------------------------------------- communicator
def make_bootstrap_allgather(group=None, device=None):
    """ctypes callback implementing adapcc_bootstrap_allgather_fn over a
    torch.distributed group (gloo: CPU tensors; nccl: tensors on `device`).
    The paper's set-up AllGather of IPC handles (Fig. 10)."""
    import torch
    import torch.distributed as dist
    n = dist.get_world_size(group)
    backend = dist.get_backend(group)
    tdev = torch.device("cuda", device if device is not None else torch.cuda.current_device()) \
        if backend == "nccl" else torch.device("cpu")

    def ag(send, recv, nbytes, _ctx):
        try:
            mine = torch.frombuffer(bytearray(ctypes.string_at(send, nbytes)), dtype=torch.uint8)
            outs = [torch.empty(nbytes, dtype=torch.uint8, device=tdev) for _ in range(n)]
            dist.all_gather(outs, mine.to(tdev), group=group)
            blob = b"".join(o.cpu().numpy().tobytes() for o in outs)
            ctypes.memmove(recv, blob, len(blob))
            return 0
        except Exception:  # noqa: BLE001 -- reported as ADAPCC_ERR_BOOTSTRAP
            return 1

    return AG_FN(ag)


def make_store_allgather(ranks, rank, store=None, tag="adapcc"):
    """ctypes all-gather callback over `ranks` only (ascending order), through
    the torch.distributed key-value store -- usable after a fault, when the
    faulty ranks cannot take part in a process-group collective (NEXT-3)."""
    import torch.distributed as dist
    store = store if store is not None else dist.distributed_c10d._get_default_store()
    ranks = sorted(ranks)
    seq = [0]

    def ag(send, recv, nbytes, _ctx):
        try:
            seq[0] += 1
            pre = f"{tag}/{seq[0]}/"
            store.set(pre + str(rank), ctypes.string_at(send, nbytes))
            keys = [pre + str(r) for r in ranks]
            store.wait(keys)
            blob = b"".join(bytes(store.get(k)) for k in keys)
            ctypes.memmove(recv, blob, len(blob))
            return 0
        except Exception:  # noqa: BLE001 -- reported as ADAPCC_ERR_BOOTSTRAP
            return 1

    return AG_FN(ag)


def coord_decide(board, nranks, members, ticket, buy_cost, cycle, timeout):
    """adapcc_coord_decide (native break-even loop; runs without
    the GIL).  board: address of the readiness board; members: rank set;
    buy_cost: nranks + 1 seconds.  Returns (full, ready set, t_first,
    t_decide) on the time.perf_counter clock; TimeoutError if nobody is ready."""
    costs = (ctypes.c_double * (nranks + 1))(*buy_cost)
    mask, full = ctypes.c_uint64(), ctypes.c_int()
    t_first, t_decide = ctypes.c_double(), ctypes.c_double()
    code = _load().adapcc_coord_decide(board, nranks, _mask(members, nranks), ticket, costs, cycle, timeout,
                                       ctypes.byref(mask), ctypes.byref(full), ctypes.byref(t_first),
                                       ctypes.byref(t_decide))
    if code == TIMEOUT:
        raise TimeoutError("no worker became ready")
    _check(code, "coord_decide")
    return bool(full.value), {r for r in range(nranks) if (mask.value >> r) & 1}, t_first.value, t_decide.value


def coord_await(board, nranks, late, ticket, phase1_event, t_first, fault_factor, timeout):
    """adapcc_coord_await (native, P:L131 / P:L139): the set of late ranks
    judged faulty (empty: all signalled, run phase 2).  phase1_event: a raw
    cudaEvent_t handle or None."""
    faulty = ctypes.c_uint64()
    code = _load().adapcc_coord_await(board, nranks, _mask(late, nranks), ticket, phase1_event,
                                      -1.0 if t_first is None else t_first, fault_factor or 0.0, timeout,
                                      ctypes.byref(faulty))
    if code == TIMEOUT:
        raise TimeoutError("late ranks never became ready (fault: set fault_factor or see exclude_faulty)")
    _check(code, "coord_await")
    return {r for r in range(nranks) if (faulty.value >> r) & 1}


class PreparedCall:
    """One collective call with its C arguments converted once (ctypes values),
    re-enqueued by calling it: the per-call host cost is one C call
    (Communicator.prepare_*).  Keeps references to the tensors it names."""

    __slots__ = ("_fn", "_args", "_where", "_keep")

    def __init__(self, fn, args, where, keep=None):
        conv = []
        for a, t in zip(args, fn.argtypes):
            conv.append(a if isinstance(a, (ctypes._SimpleCData, ctypes.Array, ctypes._Pointer)) or a is None
                        else t(a))
        self._fn, self._args, self._where, self._keep = fn, tuple(conv), where, keep

    def __call__(self):
        code = self._fn(*self._args)
        if code:
            raise AdapccError(code, self._where)


class Communicator:
    """A communicator (the paper's transmission contexts)."""

    def __init__(self, handle, nranks, rank, device, loopback, keep=None):
        self._h = handle
        self.nranks = nranks
        self.rank = rank
        self.device = device
        self.loopback = loopback
        self._keep = keep
        self.members = set(range(nranks))

    @property
    def members(self):
        return self._members

    @members.setter
    def members(self, live):
        self._members = set(live)
        self._members_mask = _mask(self._members, self.nranks)

    def _ready_mask(self, ready):
        return self._members_mask if ready is None else _mask(ready, self.nranks)

    # ---- fault tolerance (NEXT-3)
    def exclude(self, dead, store=None):
        """Exclude faulty ranks; collective over the survivors.
        Multi-process: the survivors all-gather through the distributed store."""
        dead = set(dead)
        live = self.members - dead
        mask = _mask(dead, self.nranks)
        if self.loopback:
            cb = AG_FN()
        else:
            tag = f"adapcc-exclude/{_mask(live, self.nranks)}"
            cb = make_store_allgather(live, self.rank, store, tag)
            self._keep_exclude = cb      # the library calls it again for registrations
        _check(_load().adapcc_exclude(self._h, mask, cb, None), "exclude")
        v = ctypes.c_uint64()
        _check(_load().adapcc_members(self._h, ctypes.byref(v)), "members")
        self.members = {g for g in range(self.nranks) if (v.value >> g) & 1}

    # ---- construction
    @classmethod
    def loopback(cls, nranks, device=0, scratch_bytes=0, mode="direct"):
        L = _load()
        h = ctypes.c_void_p()
        _check(L.adapcc_init_loopback(ctypes.byref(h), nranks, device, scratch_bytes, MODE[mode]),
               "init_loopback")
        return cls(h, nranks, 0, device, True)

    @classmethod
    def init(cls, group=None, scratch_bytes=0, device=None):
        """Multi-process communicator over a torch.distributed process group."""
        import torch
        import torch.distributed as dist
        L = _load()
        rank = dist.get_rank(group)
        n = dist.get_world_size(group)
        dev = torch.cuda.current_device() if device is None else device
        cb = make_bootstrap_allgather(group, dev)
        h = ctypes.c_void_p()
        _check(L.adapcc_init(ctypes.byref(h), rank, n, dev, scratch_bytes, cb, None), "init")
        return cls(h, n, rank, dev, False, keep=cb)

    # ---- control
    def set_strategy(self, coll, text, stream=None):
        s = ctypes.c_void_p(0) if stream is None else _stream(stream, self.device)
        _check(_load().adapcc_set_strategy(self._h, COLL[coll], text.encode(), s), "set_strategy")

    def config(self, key, value):
        _check(_load().adapcc_config(self._h, key.encode(), int(value)), "config")

    def get_async_error(self):
        return _load().adapcc_get_async_error(self._h)

    def launch_count(self):
        v = ctypes.c_uint64()
        _check(_load().adapcc_launch_count(self._h, ctypes.byref(v)), "launch_count")
        return v.value

    def trace(self, max_records=1 << 20):
        """Drain the in-kernel trace (enable with config("trace", capacity)).

        Returns (records, n_total): a numpy structured array with fields
        launch, cta, item, task, t0, t1, t2, bytes (include/adapcc.h,
        adapcc_trace_read) and the number of records the kernels wrote."""
        import numpy as np
        dt = np.dtype([("launch", "<u4"), ("cta", "<u4"), ("item", "<u4"), ("task", "<u4"),
                       ("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8"), ("bytes", "<u8")])
        buf = np.zeros(max_records, dtype=dt)
        n, tot = ctypes.c_uint32(), ctypes.c_uint32()
        _check(_load().adapcc_trace_read(self._h, buf.ctypes.data, max_records, ctypes.byref(n),
                                         ctypes.byref(tot)), "trace_read")
        return buf[:n.value].copy(), tot.value

    def last_engine(self):
        """Kernel of the most recent launch: 0 LDG/STG fold, 1 TMA pipeline, 3 flat kernel."""
        v = ctypes.c_int()
        _check(_load().adapcc_last_engine(self._h, ctypes.byref(v)), "last_engine")
        return v.value

    def finalize(self):
        if self._h:
            _load().adapcc_finalize(self._h)
            self._h = None

    def __del__(self):
        try:
            self.finalize()
        except Exception:  # noqa: BLE001
            pass

    # ---- multi-process collectives
    def allreduce(self, x, out=None, ready=None, accumulate=False, stream=None, late=None):
        """late: None | 'join' (phase 1) | 'complement' (phase 2); a late rank
        passes its input, read once it signalled ready (signal_ready)."""
        out = x if out is None else out
        m = self._ready_mask(ready)
        send = x if ((m >> self.rank) & 1 or late is not None) else None
        flags = (FLAG_ACCUMULATE if accumulate else 0) | _late_flag(late)
        _check(_load().adapcc_allreduce(self._h, _ptr(send), _ptr(out), out.numel(),
                                        _dtype_code(out), m, flags, _stream(stream, self.device)),
               "allreduce")
        return out

    def allgather(self, x, out, ready=None, stream=None):
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        cnt = out.numel() // self.nranks
        _check(_load().adapcc_allgather(self._h, _ptr(send), _ptr(out), cnt, _dtype_code(out), m,
                                        _stream(stream, self.device)), "allgather")
        return out

    def alltoall(self, x, out, ready=None, stream=None):
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        cnt = out.numel() // self.nranks
        _check(_load().adapcc_alltoall(self._h, _ptr(send), _ptr(out), cnt, _dtype_code(out), m,
                                       _stream(stream, self.device)), "alltoall")
        return out

    def reduce(self, x, out, root, ready=None, accumulate=False, stream=None):
        """Only the root's `out` is written (non-roots may pass None)."""
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        n_el = (out if out is not None else x).numel()
        _check(_load().adapcc_reduce(self._h, _ptr(send), _ptr(out), n_el,
                                     _dtype_code(out if out is not None else x), root, m,
                                     FLAG_ACCUMULATE if accumulate else 0, _stream(stream, self.device)), "reduce")
        return out

    def broadcast(self, x, out, root, ready=None, stream=None):
        m = self._ready_mask(ready)
        send = x if (self.rank == root and (m >> root) & 1) else None
        _check(_load().adapcc_broadcast(self._h, _ptr(send), _ptr(out), out.numel(), _dtype_code(out),
                                        root, m, _stream(stream, self.device)), "broadcast")
        return out

    def reducescatter(self, x, out, ready=None, accumulate=False, stream=None):
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        _check(_load().adapcc_reducescatter(self._h, _ptr(send), _ptr(out), out.numel(),
                                            _dtype_code(out), m, FLAG_ACCUMULATE if accumulate else 0,
                                            _stream(stream, self.device)), "reducescatter")
        return out

    # ---- zero-copy (multi-process): registered buffers, DIRECT plan over NVLink
    def register(self, t):
        """Register tensor t's storage for zero-copy collectives (collective call)."""
        rid = ctypes.c_int()
        nbytes = t.numel() * t.element_size()
        _check(_load().adapcc_register_buffer(self._h, ctypes.c_void_p(t.data_ptr()), nbytes,
                                              ctypes.byref(rid)), "register_buffer")
        regs = self.__dict__.setdefault("_regs", {})
        regs[rid.value] = (t.data_ptr(), nbytes, t)
        return rid.value

    def deregister(self, rid):
        _check(_load().adapcc_deregister_buffer(self._h, rid), "deregister_buffer")
        self.__dict__.get("_regs", {}).pop(rid, None)

    def _reg_of(self, t):
        for rid, (ptr, nbytes, _) in self.__dict__.get("_regs", {}).items():
            off = t.data_ptr() - ptr
            if 0 <= off and off + t.numel() * t.element_size() <= nbytes:
                return rid, off
        raise ValueError("tensor is not inside a registered buffer (call comm.register first)")

    def collective_zc(self, coll, x, out, count, root=0, ready=None, accumulate=False, stream=None,
                      late=None):
        """Any collective on registered tensors x / out (same offsets on every rank)."""
        sr, so = self._reg_of(x)
        rr, ro = self._reg_of(out)
        m = self._ready_mask(ready)
        flags = (FLAG_ACCUMULATE if accumulate else 0) | _late_flag(late)
        _check(_load().adapcc_collective_zc(self._h, COLL[coll], sr, so, rr, ro, count, _dtype_code(out),
                                            root, m, flags, _stream(stream, self.device)), coll + "_zc")
        return out

    # ---- loopback collectives (lists of per-virtual-rank tensors)
    def _arrays(self, xs, outs, m):
        """ctypes pointer arrays for the _lb calls, reused while the pointers repeat."""
        key = [x.data_ptr() if x is not None and (m >> r) & 1 else 0 for r, x in enumerate(xs)]
        key += [o.data_ptr() if o is not None else 0 for o in outs]
        cached = self.__dict__.get("_arr_cache")
        if cached is not None and cached[0] == key:
            return cached[1], cached[2]
        n = self.nranks
        S = (ctypes.c_void_p * n)(*key[:n])
        D = (ctypes.c_void_p * n)(*key[n:])
        self._arr_cache = (key, S, D)
        return S, D

    def _allreduce_lb_args(self, xs, outs, ready, accumulate, stream, late):
        m = self._ready_mask(ready)
        if late is not None:
            # phase 2 reads the late ranks' inputs: pass every input
            S, D = self._arrays(xs, outs, _mask(self.members, self.nranks))
        else:
            S, D = self._arrays(xs, outs, m)
        flags = (FLAG_ACCUMULATE if accumulate else 0) | _late_flag(late)
        return (self._h, S, D, outs[0].numel(), _dtype_code(outs[0]), m, flags, _stream(stream, self.device))

    def allreduce_lb(self, xs, outs, ready=None, accumulate=False, stream=None, late=None):
        """late: None | 'join' (phase 1) | 'complement' (phase 2)."""
        _check(_load().adapcc_allreduce_lb(*self._allreduce_lb_args(xs, outs, ready, accumulate, stream, late)),
               "allreduce_lb")
        return outs

    # ---- prepared calls: every argument marshalled once
    def prepare_allreduce_lb(self, xs, outs, ready=None, accumulate=False, stream=None, late=None):
        """A persistent loopback AllReduce: the returned callable enqueues the
        same call (same tensors, mask, flags and stream -- the current stream
        at prepare time unless given) with one C call and no per-call
        marshalling.  The tensors must stay alive and keep their storage."""
        return PreparedCall(_load().adapcc_allreduce_lb,
                            self._allreduce_lb_args(xs, outs, ready, accumulate, stream, late),
                            "allreduce_lb", keep=(xs, outs))

    def prepare_allreduce(self, x, out=None, ready=None, accumulate=False, stream=None):
        """A persistent multi-process AllReduce (see prepare_allreduce_lb)."""
        out = x if out is None else out
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        args = (self._h, _ptr(send), _ptr(out), out.numel(), _dtype_code(out), m,
                FLAG_ACCUMULATE if accumulate else 0, _stream(stream, self.device))
        return PreparedCall(_load().adapcc_allreduce, args, "allreduce", keep=(x, out))

    def prepare_collective_zc(self, coll, x, out, count, root=0, ready=None, accumulate=False, stream=None,
                              late=None):
        """A persistent zero-copy collective on registered tensors (see prepare_allreduce_lb)."""
        sr, so = self._reg_of(x)
        rr, ro = self._reg_of(out)
        m = self._ready_mask(ready)
        flags = (FLAG_ACCUMULATE if accumulate else 0) | _late_flag(late)
        args = (self._h, COLL[coll], sr, so, rr, ro, count, _dtype_code(out), root, m, flags,
                _stream(stream, self.device))
        return PreparedCall(_load().adapcc_collective_zc, args, coll + "_zc", keep=(x, out))

    def alltoallv_lb(self, xs, outs, counts, ready=None, stream=None):
        """counts: nranks x nranks element counts (counts[s][d] from s to d)."""
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        flat = (ctypes.c_uint64 * (self.nranks * self.nranks))(*[int(v) for row in counts for v in row])
        _check(_load().adapcc_alltoallv_lb(self._h, S, D, flat, _dtype_code(outs[0]), m, _stream(stream, self.device)),
               "alltoallv_lb")
        return outs

    def alltoallv(self, x, out, counts, ready=None, stream=None):
        m = self._ready_mask(ready)
        send = x if (m >> self.rank) & 1 else None
        flat = (ctypes.c_uint64 * (self.nranks * self.nranks))(*[int(v) for row in counts for v in row])
        _check(_load().adapcc_alltoallv(self._h, _ptr(send), _ptr(out), flat, _dtype_code(out), m,
                                        _stream(stream, self.device)), "alltoallv")
        return out

    def link_probe(self, dst, nbytes, messages=1, engine="sm", iters=20, src=-1):
        """Seconds per repetition of `messages` messages of `nbytes` from `src`
        (-1 = this rank) to every rank in `dst` at once (adapcc_link_probe);
        engine "sm" (TMA bulk copies) or "ce" (copy engines).  Multi-process:
        a collective -- every rank calls it (dst may be empty)."""
        v = ctypes.c_double()
        _check(_load().adapcc_link_probe(self._h, src, _mask(set(dst), self.nranks), nbytes, messages,
                                         {"ce": 0, "sm": 1}[engine], iters, ctypes.byref(v)), "link_probe")
        return v.value

    def ready_board(self):
        """(address, shared) of the host-mapped readiness board (adapcc_ready_board):
        word r = the ticket rank r last signalled ready for; words 64..127 are
        the coordinator's.  shared: every rank's word is visible here."""
        p, sh = ctypes.c_void_p(), ctypes.c_int()
        _check(_load().adapcc_ready_board(self._h, ctypes.byref(p), ctypes.byref(sh)), "ready_board")
        return p.value, bool(sh.value)

    def spin(self, ns, stream=None):
        """Enqueue a one-thread %globaltimer spin of `ns` nanoseconds (controlled straggler)."""
        _check(_load().adapcc_spin(self._h, int(ns), _stream(stream, self.device)), "spin")

    def nvls_setup(self, nbytes=256 << 20):
        """Multicast team + NVLS scratch (adapcc_nvls_setup, collective).
        Returns (ok, reason); ok False when the box cannot multicast."""
        why = ctypes.create_string_buffer(256)
        code = _load().adapcc_nvls_setup(self._h, nbytes, why, 256)
        if code not in (SUCCESS, UNSUPPORTED):
            raise AdapccError(code, "nvls_setup: " + why.value.decode())
        return code == SUCCESS, why.value.decode()

    def late_advance(self):
        """Consume the next ticket without a LATE_JOIN call (adapcc_late_advance)."""
        v = ctypes.c_uint64()
        _check(_load().adapcc_late_advance(self._h, ctypes.byref(v)), "late_advance")
        return v.value

    def late_ticket(self):
        v = ctypes.c_uint64()
        _check(_load().adapcc_late_ticket(self._h, ctypes.byref(v)), "late_ticket")
        return v.value

    def signal_ready(self, rank=-1, ticket=0, stream=None):
        """Mark `rank` ready for late join after the work already on `stream`."""
        _check(_load().adapcc_signal_ready(self._h, rank, ticket, _stream(stream, self.device)), "signal_ready")

    def allgather_lb(self, xs, outs, ready=None, stream=None):
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        _check(_load().adapcc_allgather_lb(self._h, S, D, outs[0].numel() // self.nranks,
                                           _dtype_code(outs[0]), m, _stream(stream, self.device)), "allgather_lb")
        return outs

    def alltoall_lb(self, xs, outs, ready=None, stream=None):
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        _check(_load().adapcc_alltoall_lb(self._h, S, D, outs[0].numel() // self.nranks,
                                          _dtype_code(outs[0]), m, _stream(stream, self.device)), "alltoall_lb")
        return outs

    def reduce_lb(self, xs, outs, root, ready=None, accumulate=False, stream=None):
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        _check(_load().adapcc_reduce_lb(self._h, S, D, outs[root].numel(), _dtype_code(outs[root]), root,
                                        m, FLAG_ACCUMULATE if accumulate else 0, _stream(stream, self.device)),
               "reduce_lb")
        return outs

    def broadcast_lb(self, xs, outs, root, ready=None, stream=None):
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        _check(_load().adapcc_broadcast_lb(self._h, S, D, outs[0].numel(), _dtype_code(outs[0]), root, m,
                                           _stream(stream, self.device)), "broadcast_lb")
        return outs

    def reducescatter_lb(self, xs, outs, ready=None, accumulate=False, stream=None):
        m = self._ready_mask(ready)
        S, D = self._arrays(xs, outs, m)
        _check(_load().adapcc_reducescatter_lb(self._h, S, D, outs[0].numel(), _dtype_code(outs[0]), m,
                                               FLAG_ACCUMULATE if accumulate else 0, _stream(stream, self.device)),
               "reducescatter_lb")
        return outs
