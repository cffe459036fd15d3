"""GPU behaviour tuples and flow lists -- TEST INFRASTRUCTURE ONLY.

Follows PAPER.md §IV-C-3 "GPU Behavior Abstraction" (Fig. 7
P:L143-144) step by step, for one reduce tree and one ready set R:

  isActive  -- the rank is ready.
  hasRecv   -- some direct predecessor (child) has data to send; "each rank
               recursively checks whether its predecessors have data to send"
               (P:L153).  Evaluated bottom-up (post-order).
  hasKernel -- set unless (1) hasRecv is not set, (2) isActive is false and
               there is only one active precedent (the rank is a pure relay),
               or (3) the synthesizer says a_{m,g} = 0.
  hasSend   -- not set when both isActive and hasRecv are false; never set at
               the root.

Reading Q3: "only one active precedent" counts the incoming
*flows*.  Without a_{m,g}=0 nodes that equals the number of sending children;
a node with a_{m,g}=0 forwards its flows individually (P:L154(3), Fig. 8(b)
P:L184, link-load model P:L196-203), so its parent sees several flows.

Flow lists: the value a node emits upward is a list of flows; a kernel node
emits one flow (its aggregate), a ready leaf emits its own tensor, a pure relay
re-emits its child's flow unchanged, an a=0 node emits its own tensor (if
ready) followed by its children's flows.  Order: own tensor first, then
sending children by ascending rank (reading Q5).
"""


def behavior(parent, ready, noagg=frozenset()):
    """Return (tuples, flows) for one tree.

    parent : list, parent[g] or -1 at the root.
    ready  : set of ready ranks R.
    noagg  : ranks with a_{m,g} = 0.
    tuples : dict g -> (isActive, hasRecv, hasKernel, hasSend) as bools.
    flows  : dict g -> list of flow descriptors, each ('in', r) -- rank r's
             own tensor -- or ('agg', k) -- the aggregate computed by kernel
             node k.  Defined for every rank; [] when nothing is emitted.
    """
    n = len(parent)
    root = parent.index(-1)
    children = {g: [c for c in range(n) if parent[c] == g] for g in range(n)}

    # post-order: children before parents (depth-first, ascending children)
    order = []

    def visit(g):
        for c in children[g]:
            visit(c)
        order.append(g)

    visit(root)

    tup = {}
    flows = {}
    for g in order:
        act = g in ready
        snd = [c for c in children[g] if tup[c][3]]          # children with hasSend
        has_recv = len(snd) > 0
        n_in = sum(len(flows[c]) for c in snd)
        agg = g not in noagg
        has_kernel = has_recv and agg and not ((not act) and n_in == 1)
        has_send = (act or has_recv) and g != root
        tup[g] = (act, has_recv, has_kernel, has_send)
        if has_kernel:
            flows[g] = [("agg", g)]
        else:
            f = [("in", g)] if act else []
            for c in snd:
                f += flows[c]
            flows[g] = f
    return tup, flows


def broadcast_tuples(parent):
    """Broadcast stage of AllReduce = the reduce tree reversed (Q8):
    every non-root receives, nobody aggregates, a rank sends iff it has
    children.  Returned as g -> (hasRecv, hasKernel, hasSend)."""
    n = len(parent)
    return {g: (parent[g] != -1, False, any(parent[c] == g for c in range(n)))
            for g in range(n)}
