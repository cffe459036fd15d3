"""Seeded synthetic inputs shared by tests, smoke() and bench.py.

Holds NONE of the method's arithmetic: only seeded random tensors and the
workload shapes of BASELINE.json's configs (DESIGN.md §5 "input recipe").
Both the oracle and the CUDA path consume these; neither is imported here.
"""

from .inputs import (rank_tensor, rank_tensors, bf16_bits_from_normal,  # noqa: F401
                     CONFIGS, GPT2XL_LAYERS, ready_set_from_mask, mask_from_set, moe_counts)
