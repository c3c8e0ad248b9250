"""SplitMix64 counter-mode payload generator.

64-bit word ``i`` of the stream with seed ``s`` is

    z  = s + (i + 1) * 0x9E3779B97F4A7C15          (mod 2**64)
    z  = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
    z  = (z ^ (z >> 27)) * 0x94D049BB133111EB
    z ^= z >> 31

stored little-endian; a payload of ``n`` bytes is the first ``n`` bytes of
that word stream (the tail truncates the last word).  The per-op seed is
``run_seed * 1_000_003 + op_index`` (mod 2**64).

This is an INPUT generator: the data path copies opaque bytes, and the
payload only has to be reproducible on both sides.  The CUDA test kernel
``gr_fill`` implements the same counter-based generator independently; the
GPU tests cross-check the two.
"""
from __future__ import annotations

import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
MASK64 = (1 << 64) - 1


def op_seed(run_seed: int, op_index: int) -> int:
    """Per-op seed (O11): run_seed * 1,000,003 + op_index, mod 2**64."""
    return (run_seed * 1_000_003 + op_index) & MASK64


def splitmix_word(seed: int, i: int) -> int:
    """Scalar reference: word ``i`` of stream ``seed`` (pure Python ints)."""
    z = (seed + (i + 1) * GOLDEN) & MASK64
    z = ((z ^ (z >> 30)) * M1) & MASK64
    z = ((z ^ (z >> 27)) * M2) & MASK64
    return z ^ (z >> 31)


def _words(seed: int, start: int, count: int) -> np.ndarray:
    idx = np.arange(start + 1, start + count + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & MASK64) + idx * np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
        z = z ^ (z >> np.uint64(31))
    return z


def payload(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """Bytes [offset, offset+n) of stream ``seed`` as a uint8 array."""
    if n <= 0:
        return np.zeros(0, dtype=np.uint8)
    w0 = offset // 8
    w1 = (offset + n + 7) // 8
    out = np.empty(0, dtype=np.uint8)
    parts = []
    step = 1 << 24  # 128 MiB of words per slab keeps peak memory bounded
    for s in range(w0, w1, step):
        cnt = min(step, w1 - s)
        parts.append(_words(seed, s, cnt).astype("<u8").view(np.uint8))
    out = np.concatenate(parts) if len(parts) > 1 else parts[0]
    lo = offset - w0 * 8
    return out[lo:lo + n]


def payload_into(buf: np.ndarray, seed: int) -> None:
    """Fill a uint8 buffer in place with the first len(buf) bytes of ``seed``."""
    buf[...] = payload(seed, buf.size)
