"""Counter-based seeded generator shared by the oracle and the harness.

This module holds NO arithmetic of the method (no norm, GEMV, attention,
message passing or scheduling). It only turns seeds into integers, following
SURVEY.md §8(c) C1 ("seeded generators — both sides implement independently
from this text"). The CUDA path has its own device implementation of the same
generator (csrc/kernels/init_weights.cu); the two never share code.

    f(z)        : z ^= z>>30; z *= 0xBF58476D1CE4E5B9; z ^= z>>27;
                  z *= 0x94D049BB133111EB; z ^= z>>31          (mod 2^64)
    draw(s, i)  = f(s + (i+1)*0x9E3779B97F4A7C15)   (i-th splitmix64 output)
    key(s, st)  = draw(s ^ draw(st, 0), 0)
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_MASK = (1 << 64) - 1


def mix(z: np.ndarray) -> np.ndarray:
    """The splitmix64 finaliser f(z) on a uint64 array (wrapping arithmetic)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z ^ (z >> np.uint64(30))
        z = z * _M1
        z = z ^ (z >> np.uint64(27))
        z = z * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def draw(seed, i) -> np.ndarray:
    """draw(seed, i) for array-like seed / i (broadcast), uint64 result."""
    seed = np.asarray(seed, dtype=np.uint64)
    i = np.asarray(i, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return mix(seed + (i + np.uint64(1)) * GOLDEN)


def draw_int(seed: int, i: int) -> int:
    """Scalar draw with Python ints (used by the slow reference paths)."""
    z = (seed + (i + 1) * 0x9E3779B97F4A7C15) & _MASK
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & _MASK
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & _MASK
    z ^= z >> 31
    return z


def key(seed: int, stream: int) -> int:
    """key(seed, stream) = draw(seed ^ draw(stream, 0), 0)."""
    return draw_int((seed & _MASK) ^ draw_int(stream & _MASK, 0), 0)


def splitmix64_sequence(seed: int, n: int) -> list[int]:
    """First n outputs of splitmix64 seeded with `seed` (= draw(seed, 0..n-1))."""
    return [draw_int(seed, i) for i in range(n)]


# ---------------------------------------------------------------------------
# Value encodings. Both are exact in bf16 by construction.
# ---------------------------------------------------------------------------

def _levels(seed: int, tid: int, n: int, offset: int, shift: int, bias: int) -> np.ndarray:
    """(draw(key(seed, tid), i) >> shift) - bias for i = offset..offset+n-1, int16.

    Same definition as `draw`, evaluated in 1 Mi-element chunks with in-place
    uint64 ufuncs on a small thread pool (numpy releases the GIL): a 7B layer's
    202 M draws take ~1 s instead of ~11 s (pinned against `draw` by a test)."""
    k = np.uint64(key(seed, tid))
    out = np.empty(n, dtype=np.int16)
    chunk = 1 << 20

    def run(s0: int) -> None:
        m = min(chunk, n - s0)
        z = np.arange(offset + s0 + 1, offset + s0 + m + 1, dtype=np.uint64)
        t = np.empty_like(z)
        with np.errstate(over="ignore"):
            np.multiply(z, GOLDEN, out=z)
            np.add(z, k, out=z)
            np.right_shift(z, np.uint64(30), out=t)
            np.bitwise_xor(z, t, out=z)
            np.multiply(z, _M1, out=z)
            np.right_shift(z, np.uint64(27), out=t)
            np.bitwise_xor(z, t, out=z)
            np.multiply(z, _M2, out=z)
            np.right_shift(z, np.uint64(31), out=t)
            np.bitwise_xor(z, t, out=z)
            np.right_shift(z, np.uint64(shift), out=z)
        np.subtract(z.astype(np.int16), np.int16(bias), out=out[s0:s0 + m])

    starts = range(0, n, chunk)
    if n <= chunk:
        for s0 in starts:
            run(s0)
    else:
        from concurrent.futures import ThreadPoolExecutor
        import os
        with ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 1)) as ex:
            list(ex.map(run, starts))
    return out


def weight_levels(seed: int, tid: int, n: int, offset: int = 0) -> np.ndarray:
    """int8 level k_i = (draw(key(seed, tid), i) >> 56) - 128 of weight tensor `tid`."""
    return _levels(seed, tid, n, offset, 56, 128).astype(np.int8)


def weight_values(seed: int, tid: int, n: int, offset: int = 0) -> np.ndarray:
    """Elements offset..offset+n-1 of weight tensor `tid`, as float32.

    w_i = ((draw(key(seed, tid), i) >> 56) - 128) * 2^-12   (int8 level, bf16-exact)
    """
    return _levels(seed, tid, n, offset, 56, 128).astype(np.float32) * np.float32(2.0 ** -12)


def gain_values(seed: int, tid: int, n: int) -> np.ndarray:
    """Norm gain: g_i = 1 + ((draw(key(seed, tid), i) >> 60) - 8) * 2^-6."""
    lvl = _levels(seed, tid, n, 0, 60, 8)
    return (np.float32(1.0) + lvl.astype(np.float32) * np.float32(2.0 ** -6)).astype(np.float32)
