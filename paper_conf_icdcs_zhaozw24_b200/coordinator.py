"""Relay coordinator: wait-or-proceed decisions and fault marking (NEXT-1 / NEXT-3).

Host-side policy of AdapCC's adaptive relay control (§IV-C):

* Decision cycles: every `cycle` the coordinator either keeps
  waiting for all workers or starts *phase 1* -- a partial collective among
  the ready workers, non-ready ones acting as relays -- followed by *phase 2*
  once the late workers are ready.
* Ski rental: waiting costs 1 per cycle (here: the cycle's
  duration); "buying" costs the estimated phase-1 + phase-2 time.  The
  break-even rule waits "at most until the accumulated waiting cost exceeds
  the buying cost in a time cycle", which is 2-competitive.  The time of a
  collective is estimated as S / B: S = 2(N-1) x tensor for
  AllReduce, N x tensor for AlltoAll, tensor for Broadcast, with N the
  participating workers; B = aggregate profiled link bandwidth of the graph.
* Fault tolerance: after phase 1 completes, workers still not ready
  after T_fault = 5 x (time since the fastest worker became ready) are marked
  faulty and excluded.

On B200 the cycle is scaled from the paper's 5 ms to the collective's own
time scale (µs), see DESIGN.md §3 reading R2.  The coordinator is pure host
logic; it produces the ready masks the engine consumes.
"""

from dataclasses import dataclass, field

T_FAULT_FACTOR = 5.0


def comm_volume(coll, n_participants, tensor_bytes):
    """S of P:L135 for N participating workers."""
    if n_participants <= 1:
        return 0.0
    if coll == "allreduce":
        return 2.0 * (n_participants - 1) * tensor_bytes
    if coll == "alltoall":
        return float(n_participants) * tensor_bytes
    if coll == "broadcast":
        return float(tensor_bytes)
    raise ValueError(coll)


def collective_time(coll, n_participants, tensor_bytes, aggregate_bw):
    """S / B estimate of one collective; aggregate_bw in bytes/s."""
    return comm_volume(coll, n_participants, tensor_bytes) / aggregate_bw


@dataclass
class Decision:
    action: str                 # 'wait' | 'full' | 'phase1'
    time: float                 # when the decision is taken
    ready: frozenset = frozenset()
    relays: frozenset = frozenset()


@dataclass
class Coordinator:
    """Break-even (ski-rental) coordinator for one collective at a time.

    n            : number of workers
    coll         : 'allreduce' | 'alltoall' | 'broadcast'
    tensor_bytes : bytes per worker
    link_bw      : bandwidth of one link (bytes/s); the aggregate bandwidth
                   B of a collective among k workers is k * link_bw (every
                   GPU's NVSwitch port, "accumulating the profiled link
                   bandwidth in the communication graph")
    cycle        : decision period (seconds)
    """
    n: int
    coll: str
    tensor_bytes: float
    link_bw: float
    cycle: float
    waited: float = 0.0
    history: list = field(default_factory=list)

    def _t(self, k):
        return collective_time(self.coll, k, self.tensor_bytes, max(k, 1) * self.link_bw)

    def buy_cost(self, ready_count):
        """Estimated phase 1 (ready workers) + phase 2 (late workers) time."""
        late = self.n - ready_count
        phase2 = self._t(late + 1) if late else 0.0   # late data reaches the others
        return self._t(ready_count) + phase2

    def full_cost(self):
        return self._t(self.n)

    def step(self, now, ready):
        """One decision cycle at time `now` with the set of ready workers."""
        ready = frozenset(ready)
        if len(ready) == self.n:
            d = Decision("full", now, ready)
        elif ready and self.waited + self.cycle > self.buy_cost(len(ready)):
            # waiting one more cycle would exceed the buying cost: buy (phase 1)
            d = Decision("phase1", now, ready, frozenset(range(self.n)) - ready)
        else:
            self.waited += self.cycle
            d = Decision("wait", now, ready)
        self.history.append(d)
        return d

    def run(self, arrivals, start=0.0):
        """Drive cycles over known arrival times (simulation / tests).

        arrivals: list of per-worker ready times.  Returns (decision, finish
        time): phase 1 starts at the decision, phase 2 starts once the last
        worker is ready and phase 1 is done; a full collective starts when all
        are ready.  Competitive analysis: finish - first arrival vs OPT."""
        t = start
        while True:
            ready = {r for r, a in enumerate(arrivals) if a <= t}
            d = self.step(t, ready)
            if d.action == "full":
                return d, t + self.full_cost()
            if d.action == "phase1":
                p1_end = t + self._t(len(ready))
                late_end = max(arrivals)
                p2 = self._t(self.n - len(ready) + 1)
                return d, max(p1_end, late_end) + p2
            t += self.cycle


def offline_optimum(arrivals, n, coll, tensor_bytes, link_bw, cycle):
    """OPT: the best decision time in hindsight (any cycle boundary)."""
    c = Coordinator(n, coll, tensor_bytes, link_bw, cycle)
    last = max(arrivals)
    best = last + c.full_cost()  # wait for everyone
    t = 0.0
    while t < last:
        ready = [r for r, a in enumerate(arrivals) if a <= t]
        if ready:
            p1_end = t + c._t(len(ready))
            best = min(best, max(p1_end, last) + c._t(n - len(ready) + 1))
        t += cycle
    return best


def faulty_workers(ready_times, phase1_end, now, factor=T_FAULT_FACTOR):
    """after phase 1, workers not ready within T_fault = factor x (time
    since the fastest worker became ready) are faulty.  ready_times: dict
    worker -> ready time, or None if not ready yet."""
    first = min(t for t in ready_times.values() if t is not None)
    t_fault = factor * (phase1_end - first)
    if now - phase1_end < t_fault:
        return set()
    return {r for r, t in ready_times.items() if t is None}


def exclude_faulty(comm, ready_times, phase1_end, now, factor=T_FAULT_FACTOR, store=None):
    """P:L139-146 end to end: identify the faulty workers with the T_fault rule
    and exclude them from the communicator (adapcc_exclude), after which the
    survivors continue on the same arenas with the survivors' default
    strategy.  Returns the set excluded (empty: nothing to do yet)."""
    faulty = faulty_workers(ready_times, phase1_end, now, factor) & set(comm.members)
    if faulty:
        comm.exclude(faulty, store=store)
    return faulty


# ------------------------------------------------------- online coordinator
BOARD_DECISION = 64      # readiness-board words: 64 sequence, 65 action, 66 mask (adapcc_ready_board)
BOARD_PHASE2 = 68        # 68 sequence, 69 faulty mask (0: every late rank signalled, run phase 2)
_ACTIONS = {"full": 1, "phase1": 2}


class ReadyBoard:
    """Host view of the communicator's readiness board (adapcc_ready_board):
    word r holds the ticket rank r last signalled ready for, written by the
    device (system-scope release) right after the rank's computation; the
    decision area carries the leader's decisions to the other ranks of the
    node.  Reads are plain host loads -- no device round trip (the
    coordinator "receives communication requests from each worker")."""

    def __init__(self, comm):
        import ctypes
        addr, self.shared = comm.ready_board()
        self.addr = addr
        self.n = comm.nranks
        self.words = (ctypes.c_uint64 * 128).from_address(addr)

    def ready(self, ticket):
        w = self.words
        return frozenset(r for r in range(self.n) if w[r] >= ticket)

    def publish(self, seq, action, mask):
        w = self.words
        w[BOARD_DECISION + 1] = _ACTIONS[action]
        w[BOARD_DECISION + 2] = mask
        w[BOARD_DECISION] = seq            # last: followers read seq first (x86 stores stay ordered)

    def publish_phase2(self, seq, faulty):
        w = self.words
        w[BOARD_PHASE2 + 1] = faulty
        w[BOARD_PHASE2] = seq

    def wait_phase2(self, seq, timeout, clock):
        """Follower side of the phase-2 decision; returns the faulty mask."""
        w = self.words
        t0 = clock()
        while w[BOARD_PHASE2] < seq:
            if clock() - t0 > timeout:
                raise TimeoutError("coordinator phase-2 decision not published")
        return int(w[BOARD_PHASE2 + 1])

    def wait_decision(self, seq, timeout, clock):
        w = self.words
        t0 = clock()
        while w[BOARD_DECISION] < seq:
            if clock() - t0 > timeout:
                raise TimeoutError("coordinator decision not published")
        action = {v: k for k, v in _ACTIONS.items()}[int(w[BOARD_DECISION + 1])]
        return action, int(w[BOARD_DECISION + 2])


class OnlineCoordinator:
    """The relay coordinator on the hot path: one AllReduce per
    call, driven by real readiness.

    Every decision cycle the leader (rank 0, or the loopback process) reads
    the readiness board -- which ranks signalled this collective's ticket --
    and applies the break-even rule (the native loop adapcc_coord_decide, with
    the policy's buy_cost per ready count); it publishes "full"
    (everyone ready) or "phase1" (ready ranks aggregate, the others relay) on
    the board, and every rank issues the same LATE_JOIN call with that mask
    (late ranks' chunks still join the ongoing aggregation chunk by chunk,
    P:L131).  Each rank then polls the board until every late rank signalled
    and issues LATE_COMPLEMENT (phase 2: only the chunks phase 1 missed).

    issue(mask, late) enqueues this rank's collective call: late = None (a
    plain collective over everyone: the "full" decision, after which the
    round's ticket is retired with adapcc_late_advance), 'join' (phase 1) or
    'complement' (phase 2).  The callback decides what a phase is, so the
    same coordinator drives AlltoAll / Broadcast too (phase 1 = the ready
    sources, phase 2 = the late ones; P:L135 prices them with the policy's
    `coll`).  Ranks signal readiness with comm.signal_ready(ticket=
    coordinator.ticket()) after their computation (the ticket of the
    collective the coordinator runs next).  policy_factory() returns a
    Coordinator (its buy_cost(k) table drives the decision); cycle: seconds
    between decisions (the paper's 5 ms, scaled to the collective's time
    scale, reading R2).  The waiting loops are native (adapcc_coord_decide /
    adapcc_coord_await: plain host loads of the board, no interpreter lock
    held) and time with CLOCK_MONOTONIC, the clock of time.perf_counter."""

    def __init__(self, comm, policy_factory, cycle=5e-6, timeout=30.0, fault_factor=None,
                 store=None, stream=None):
        """fault_factor: apply the T_fault rule -- late ranks not
        ready fault_factor x (phase-1 end - first ready) after phase 1 ended
        are faulty: the survivors exclude them (adapcc_exclude; multi-process
        through `store`) and keep the phase-1 result.  None: wait
        for them up to `timeout`.  stream: the stream issue() enqueues phase 1
        on (its end is T_fault's reference; default: the current stream)."""
        import time
        self.fault_factor = fault_factor
        self.store = store
        self.stream = stream
        self.comm = comm
        self.board = ReadyBoard(comm)
        self.policy_factory = policy_factory
        self.cycle = cycle
        self.timeout = timeout
        self.clock = time.perf_counter
        self.seq = 0
        self.leader = comm.loopback or comm.rank == 0
        if not comm.loopback and comm.nranks > 1 and not self.board.shared:
            raise RuntimeError("online coordinator needs a node-shared readiness board (POSIX shared memory)")

    def ticket(self):
        """Ticket of the next collective (its phase 1 is the next LATE_JOIN call)."""
        return self.comm.late_ticket() + 1

    def allreduce(self, issue):
        n, clock = self.comm.nranks, self.clock
        members = getattr(self.comm, "members", None) or set(range(n))
        all_mask = sum(1 << r for r in members)        # excluded ranks take no part
        t = self.ticket()
        self.seq += 1
        t0 = clock()
        t_first = None
        if self.leader:
            from . import adapcc as A
            policy = self.policy_factory()
            if len(members) < n and hasattr(policy, "n"):
                policy.n = len(members)        # the policy prices the survivors' collective
            costs = [float("inf")] + [policy.buy_cost(k) for k in range(1, n + 1)]
            full, ready, t_first, _ = A.coord_decide(self.board.addr, n, members, t, costs, self.cycle,
                                                     self.timeout)
            action = "full" if full else "phase1"
            mask = all_mask if full else sum(1 << r for r in ready)
            if not self.comm.loopback:
                self.board.publish(self.seq, action, mask)
        else:
            action, mask = self.board.wait_decision(self.seq, self.timeout, clock)
        t_decide = clock()
        if action == "full":                  # nobody is late: the plain (fastest) plan
            self.comm.late_advance()          # ... and this round's signals are retired
            issue(mask, None)
        else:
            issue(mask, "join")               # phase 1
            self._p1_done = self._record()
            if self.comm.late_ticket() < t:   # (a phase 1 that is not a LATE_JOIN call, e.g. AlltoAll)
                self.comm.late_advance()
        late = all_mask & ~mask
        t_late = None
        faulty = 0
        if late:
            faulty = self._phase2_or_fault(t, mask, late, t0, t_first)
            if not faulty:
                t_late = clock()
                issue(mask, "complement")
            else:   # T_fault passed: the survivors keep the phase-1 result and drop the faulty ranks
                dead = {r for r in range(n) if (faulty >> r) & 1}
                if self.comm.loopback or self.comm.rank not in dead:
                    self.comm.exclude(dead, store=self.store)
        return {"action": action, "mask": mask, "ticket": t, "decided_after_s": t_decide - t0,
                "phase2_after_s": None if t_late is None else t_late - t0,
                "faulty": sorted(r for r in range(n) if (faulty >> r) & 1)}

    def _phase2_or_fault(self, t, mask, late, t0, t_first):
        """Leader: wait until every late rank signalled (-> 0) or, with a
        fault_factor, until T_fault after phase 1 passes (-> the mask of the
        late ranks still not ready); publish it.  Followers: read it."""
        from . import adapcc as A
        n = self.comm.nranks
        self.seq2 = getattr(self, "seq2", 0) + 1
        if not self.leader:
            return self.board.wait_phase2(self.seq2, self.timeout, self.clock)
        ev = self._p1_done
        dead = A.coord_await(self.board.addr, n, {r for r in range(n) if (late >> r) & 1}, t,
                             None if ev is None else ev.cuda_event, t_first, self.fault_factor,
                             max(self.timeout - (self.clock() - t0), 0.0))
        faulty = sum(1 << r for r in dead)
        if not self.comm.loopback:
            self.board.publish_phase2(self.seq2, faulty)
        return faulty

    def _record(self):
        """A CUDA event after phase 1 on the issue stream (None without a GPU:
        host-only tests treat phase 1 as ended when issue() returns)."""
        try:
            import torch
        except ImportError:
            return None
        if not torch.cuda.is_available():
            return None
        ev = torch.cuda.Event()
        ev.record(self.stream)
        return ev
