"""PyTorch DDP communication hook backed by the AdapCC engine (NEXT-4).

The paper exposes "a communication hook for PyTorch DDP".  Usage:

    comm = Communicator.init(group)              # one per process
    ddp.register_comm_hook(AdapccHookState(comm), adapcc_allreduce_hook)

Each gradient bucket is averaged in place by one engine launch on the current
stream (the STAGED protocol, or the zero-copy DIRECT plan when the bucket's
storage was registered with comm.register).  With auto_register=True the hook
registers every bucket buffer the first time it sees it, so a training loop
runs zero-copy from its first step without touching DDP internals.  DDP
launches buckets in index order on every rank, which keeps the collective
registrations in the same order everywhere; DDP rebuilds its buckets once
after the first iteration, so each bucket is registered at most twice.
`ready` may restrict the aggregation to the ready ranks (partial
aggregation); the bucket is then divided by the number of contributing ranks.

With a coordinator (coordinator.OnlineCoordinator, NEXT-1 P:L129-137) the
hook signals this rank's readiness for the bucket (its gradients are complete
on the current stream) and lets the coordinator decide: everyone ready -> one
plain AllReduce; otherwise phase 1 among the ready ranks with late join, then
phase 2 once the late ranks signalled.  Every bucket ends with the full sum
(the paper's model-update consistency), divided by every rank.  The
collective runs on its own stream, NOT ordered after this rank's computation:
a late rank still launches phase 1 right away and its chunks join as its
ready signal lands ("asynchronously participate ... as relays"); the
bucket is staged into a per-bucket input buffer (after the gradients, on the
compute stream, before the signal) and the result lands in a per-bucket
output buffer that the compute stream copies back after phase 2.  A rank is
only in a decision's ready mask once its signal reached the board, i.e. after
its staged input is complete.
"""

import torch


class AdapccHookState:
    def __init__(self, comm, ready=None, auto_register=False, coordinator=None):
        self.comm = comm
        self.ready = ready            # None = every rank
        self.auto_register = auto_register
        self.coordinator = coordinator
        self.registered = 0           # buffers this hook registered
        self.zero_copy_calls = 0
        self.staged_calls = 0
        self.decisions = []           # coordinator: one result dict per bucket
        self._inputs = {}             # coordinator: staged input / output per bucket buffer
        self._stream = None           # coordinator: the collective's own stream

    def contributors(self):
        if self.ready is None:              # every live rank (all, unless some were excluded)
            return len(self.comm.members)
        if isinstance(self.ready, int):
            return bin(self.ready).count("1")
        return len(set(self.ready))


def _coordinated(state, buf):
    comm, coord = state.comm, state.coordinator
    key = (buf.data_ptr(), buf.numel(), buf.dtype)
    xy = state._inputs.get(key)
    if xy is None:
        xy = state._inputs[key] = (torch.empty_like(buf), torch.empty_like(buf))
    x, y = xy
    if state._stream is None:
        state._stream = torch.cuda.Stream(priority=-1)
    cur, cs = torch.cuda.current_stream(), state._stream
    x.copy_(buf)                                  # after this rank's gradients (compute stream)
    comm.signal_ready(ticket=coord.ticket())      # ... then the ready signal
    res = coord.allreduce(lambda mask, late: comm.allreduce(x, y, ready=mask, late=late, stream=cs))
    done = torch.cuda.Event()
    done.record(cs)
    cur.wait_event(done)                          # the compute stream resumes after phase 2
    buf.copy_(y).div_(len(comm.members))
    state.decisions.append(res)
    state.staged_calls += 1 + (res["phase2_after_s"] is not None)
    fut = torch.futures.Future()
    fut.set_result(buf)
    return fut


def adapcc_allreduce_hook(state, bucket):
    buf = bucket.buffer()
    comm = state.comm
    if state.coordinator is not None:
        return _coordinated(state, buf)
    try:
        comm._reg_of(buf)
        registered = True
    except ValueError:
        registered = False
    if not registered and state.auto_register:
        comm.register(buf)   # collective: every rank reaches this bucket in the same order
        state.registered += 1
        registered = True
    if registered:
        comm.collective_zc("allreduce", buf, buf, buf.numel(), ready=state.ready)
        state.zero_copy_calls += 1
    else:                # bucket not registered: STAGED protocol through the arenas
        comm.allreduce(buf, buf, ready=state.ready)
        state.staged_calls += 1
    buf.div_(state.contributors())
    fut = torch.futures.Future()
    fut.set_result(buf)
    return fut
