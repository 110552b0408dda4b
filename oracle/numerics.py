"""bf16 rounding used at the one activation rounding point (KV cache write).

SURVEY.md §8(c) C2: "Kc[l][t] = bf16_rne(k); Vc[l][t] = bf16_rne(v) (ONLY
activation rounding point)"; ambiguity register A16 (paper silent on KV
precision; §5.2 P:219 implies <=16-bit storage, A3).

Written out with integer bit operations (the textbook definition of
round-to-nearest-even on the top 16 bits of an IEEE binary32), pinned against
torch's float32->bfloat16 conversion in tests/test_oracle_numerics.py.
"""
from __future__ import annotations

import numpy as np


def bf16_rne(x) -> np.ndarray:
    """Round float32 values to bfloat16 (RNE), returned as float32.

    Input of any float dtype is first rounded to float32 (the kernel's
    precision for this decision, per the task rules: both sides round from the
    same fp32 value).
    """
    f = np.asarray(x, dtype=np.float32)
    u = f.view(np.uint32).astype(np.uint64)
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    rounded = (u + np.uint64(0x7FFF) + lsb) >> np.uint64(16)
    nan = np.isnan(f)
    out = (rounded << np.uint64(16)).astype(np.uint32)
    out = np.where(nan, np.uint32(0x7FC00000), out)
    return out.view(np.float32)


def is_bf16_exact(x) -> bool:
    f = np.asarray(x, dtype=np.float32)
    return bool(np.all((f.view(np.uint32) & np.uint32(0xFFFF)) == 0))
