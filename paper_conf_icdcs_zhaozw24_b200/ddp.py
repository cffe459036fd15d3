"""PyTorch DDP communication hook backed by the AdapCC engine (NEXT-4).

The paper exposes "a communication hook for PyTorch DDP".  Usage:

    comm = Communicator.init(group)              # one per process
    ddp.register_comm_hook(AdapccHookState(comm), adapcc_allreduce_hook)

Each gradient bucket is averaged in place by one engine launch on the current
stream (the STAGED protocol, or the zero-copy DIRECT plan when the bucket's
storage was registered with comm.register).  `ready` may restrict the
aggregation to the ready ranks (partial aggregation); the bucket is then
divided by the number of contributing ranks.
"""

import torch


class AdapccHookState:
    def __init__(self, comm, ready=None):
        self.comm = comm
        self.ready = ready            # None = every rank

    def contributors(self):
        if self.ready is None:              # every live rank (all, unless some were excluded)
            return len(self.comm.members)
        if isinstance(self.ready, int):
            return bin(self.ready).count("1")
        return len(set(self.ready))


def adapcc_allreduce_hook(state, bucket):
    buf = bucket.buffer()
    comm = state.comm
    try:
        comm._reg_of(buf)
        comm.collective_zc("allreduce", buf, buf, buf.numel(), ready=state.ready)
    except ValueError:   # bucket not registered: STAGED protocol through the arenas
        comm.allreduce(buf, buf, ready=state.ready)
    buf.div_(state.contributors())
    fut = torch.futures.Future()
    fut.set_result(buf)
    return fut
