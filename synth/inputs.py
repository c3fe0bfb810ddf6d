"""Seeded input generators (see synth/__init__.py for what may and may not live here)."""
from __future__ import annotations

import numpy as np

# Graph500 R-MAT quadrant probabilities (a, b, c; d = 1 - a - b - c), SURVEY.md §8(d) C3.
RMAT_ABC = (0.57, 0.19, 0.19)


def uniform_f32(shape, seed: int, lo: float = 0.0, hi: float = 1.0) -> np.ndarray:
    """fp32 array ~ U[lo, hi) from numpy's PCG64 stream `seed` (values never affect events)."""
    rng = np.random.default_rng(seed)
    return rng.uniform(lo, hi, size=shape).astype(np.float32)


def rmat_csr(scale: int, edge_factor: int = 16, seed: int = 3, abc=RMAT_ABC):
    """R-MAT graph on 2**scale vertices with edge_factor * 2**scale generated edges.

    Each edge picks one quadrant per bit level with probabilities (a, b, c, d). The edge list is then
    symmetrised, self-loops and duplicates are removed, and it is returned as CSR
    (rowptr int32[n+1], col int32[m]) with each row's neighbours sorted ascending.
    """
    n = 1 << scale
    m = edge_factor * n
    rng = np.random.default_rng(seed)
    a, b, c = abc
    src = np.zeros(m, dtype=np.int64)
    dst = np.zeros(m, dtype=np.int64)
    for lvl in range(scale):
        u = rng.random(m)
        bit_src = (u >= a + b).astype(np.int64)                       # quadrants c, d
        bit_dst = (((u >= a) & (u < a + b)) | (u >= a + b + c)).astype(np.int64)  # quadrants b, d
        src |= bit_src << lvl
        dst |= bit_dst << lvl
    keep = src != dst
    src, dst = src[keep], dst[keep]
    s = np.concatenate([src, dst])
    d = np.concatenate([dst, src])
    key = np.unique(s * n + d)
    s = key // n
    d = key % n
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rowptr, s + 1, 1)
    rowptr = np.cumsum(rowptr)
    return rowptr.astype(np.int32), d.astype(np.int32)


def bfs_source(rowptr: np.ndarray) -> int:
    """Max-degree vertex, lowest id on ties."""
    deg = np.diff(rowptr.astype(np.int64))
    return int(np.argmax(deg))
