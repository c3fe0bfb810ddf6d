"""splitmix64 finaliser and the counter-based generator R(i, f) — docs/EVENT_MODEL.md §3.5.

Written out step by step; numpy uint64 arithmetic wraps modulo 2**64 exactly like the spec.
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15
SEED = 0x4E5642544E564254  # "NVBTNVBT"
FSTEP = 0xD1B54A32D192ED03


def mix64_int(z: int) -> int:
    """Python-int version (exact by construction)."""
    z = (z + GOLDEN) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def mix64(z):
    """numpy uint64 version (arrays or scalars)."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def K(f: int, seed: int = SEED) -> int:
    """K(f) = mix64(SEED ^ (f * 0xD1B54A32D192ED03))."""
    return mix64_int(seed ^ ((f * FSTEP) & M64))


def R(i, f: int, seed: int = SEED):
    """R(i, f) = mix64(K(f) ^ i) for an array (or scalar) of event indices i."""
    return mix64(np.uint64(K(f, seed)) ^ np.asarray(i, dtype=np.uint64))
