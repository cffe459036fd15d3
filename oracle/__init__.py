"""AdapCC CPU oracle -- TEST INFRASTRUCTURE ONLY.

This package is the plain, slow, obviously-correct CPU definition of what the
AdapCC hot path computes (AllReduce / AllGather / AlltoAll executed along a
strategy of weighted trees under a ready-rank mask, §IV-C, §IV-D,
§V).  It is written from the paper (``/root/reference/PAPER.md``, cited as
``P:L<line>``) and from the readings listed in DESIGN.md §3.

Rules:
  * Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
    ``cpu_baseline`` / ``--impl reference`` legs may import anything here.
  * It shares no code with the CUDA path (``paper_conf_icdcs_zhaozw24_b200``):
    its own strategy parser, its own tuple derivation, its own partition rule,
    its own bf16 rounding.  Neither side imports the other.
  * Inputs come from ``synth/`` (seeded generators, no method arithmetic).

Modules:
  strategy     -- strategy text v1 parser/validator, ring expansion,
                  partition (Q9) and chunk split (Q10).
  tuples       -- GPU behaviour tuple <isActive,hasRecv,hasKernel,hasSend>
                   and the flow lists it implies (P:L154(3)).
  bf16         -- bit-level bf16 <-> fp32 with round-to-nearest-even.
  collectives  -- allreduce (replay of the strategy's reduction order and the
                  fp64 definition), allgather, alltoall.
  loads        -- AlltoAll flow routes (eq. 1) and link loads N_ij.

Parity status of every function is in DESIGN.md §4 ("pins"); there is no
function here without a pin.
"""

from . import bf16, strategy, tuples, collectives, loads  # noqa: F401
