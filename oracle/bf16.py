"""bf16 <-> fp32 conversions for the oracle (TEST INFRASTRUCTURE ONLY).

bf16 values are held as ``numpy.uint16`` bit patterns (numpy has no bf16).
The paper is silent on bf16 (reading Q6 in DESIGN.md §3): the wire format is
bf16, each aggregating node widens to fp32, adds in order and rounds ONCE with
round-to-nearest-even.  This module is the rounding definition.

Pinned by tests/test_oracle_bf16.py against ``ml_dtypes.bfloat16`` (an
independent library implementation of the same IEEE-style RNE) on exhaustive
tie/boundary patterns and random patterns.
"""

import numpy as np


def to_f32(b):
    """bf16 bits (uint16) -> float32, exact (bf16 is the top half of fp32)."""
    b = np.asarray(b, dtype=np.uint16)
    return (b.astype(np.uint32) << np.uint32(16)).view(np.float32)


def from_f32_rne(x):
    """float32 -> bf16 bits with round-to-nearest-even.

    u = bits(x); u += 0x7FFF + ((u >> 16) & 1); result = u >> 16.
    NaN is mapped to the quiet NaN 0x7FC0 with the input's sign (the test
    data never contains NaN, reading Q16).
    """
    x = np.asarray(x, dtype=np.float32)
    u = x.view(np.uint32).astype(np.uint64)          # widen: no wrap on +0x7FFF
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    r = ((u + np.uint64(0x7FFF) + lsb) >> np.uint64(16)).astype(np.uint16)
    nan = np.isnan(x)
    if np.any(nan):
        sign = ((u >> np.uint64(16)) & np.uint64(0x8000)).astype(np.uint16)
        r = np.where(nan, sign | np.uint16(0x7FC0), r).astype(np.uint16)
    return r
