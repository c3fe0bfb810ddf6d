"""Trace records and multiset digests — docs/EVENT_MODEL.md §5."""
from __future__ import annotations

import numpy as np

from .mix import mix64, mix64_int

RECORD_BYTES = 288
RECORD_DTYPE = np.dtype([
    ("launch", "<u4"), ("warp", "<u4"), ("seq", "<u4"), ("pc", "<u4"),
    ("A", "<u4"), ("P", "<u4"), ("opcode", "<u2"), ("width", "u1"), ("kind", "u1"),
    ("reserved", "<u4"), ("addr", "<u8", (32,)),
])
assert RECORD_DTYPE.itemsize == RECORD_BYTES

C1 = np.array([mix64_int(0x1000 + j) | 1 for j in range(36)], dtype=np.uint64)
C2 = np.array([mix64_int(0x2000 + j) | 1 for j in range(36)], dtype=np.uint64)


def build_records(launch, warp, seq, pc, A, P, prog, addr, E):
    """One 288-byte record per event (all arguments are per-event arrays except launch/prog).

    addr[l] is kept for lanes of E and zeroed otherwise (reading R-13)."""
    n = len(warp)
    rec = np.zeros(n, dtype=RECORD_DTYPE)
    rec["launch"] = launch
    rec["warp"] = warp
    rec["seq"] = seq
    rec["pc"] = pc
    rec["A"] = A
    rec["P"] = P
    rec["opcode"] = prog["opcode"][pc]
    rec["width"] = prog["width"][pc]
    rec["kind"] = prog["kind"][pc]
    act = ((np.asarray(E, dtype=np.uint64)[:, None] >> np.arange(32, dtype=np.uint64)[None, :]) & np.uint64(1)) == 1
    rec["addr"] = np.where(act, np.asarray(addr, dtype=np.uint64), np.uint64(0))
    return rec.view(np.uint8).reshape(n, RECORD_BYTES)


def record_hashes(recs_u8):
    """(h1, h2) per record: h_k = Σ_j x[j] · C_k[j] mod 2**64 over the 36 little-endian words."""
    x = np.ascontiguousarray(recs_u8).view("<u8").reshape(-1, 36)
    with np.errstate(over="ignore"):
        h1 = (x * C1[None, :]).sum(axis=1, dtype=np.uint64)
        h2 = (x * C2[None, :]).sum(axis=1, dtype=np.uint64)
    return h1, h2


class Digest:
    """N_rec, D1 = Σ mix64(h1), D2 = Σ mix64(h2) (all mod 2**64)."""

    def __init__(self):
        self.n = 0
        self.d1 = 0
        self.d2 = 0

    def update(self, recs_u8):
        if len(recs_u8) == 0:
            return
        h1, h2 = record_hashes(recs_u8)
        with np.errstate(over="ignore"):
            s1 = int(mix64(h1).sum(dtype=np.uint64))
            s2 = int(mix64(h2).sum(dtype=np.uint64))
        self.n += len(recs_u8)
        self.d1 = (self.d1 + s1) & ((1 << 64) - 1)
        self.d2 = (self.d2 + s2) & ((1 << 64) - 1)


def sort_records(recs_u8):
    """Canonical order for multiset comparison (R-12): by (launch, warp, seq)."""
    r = np.ascontiguousarray(recs_u8).view(RECORD_DTYPE).reshape(-1)
    order = np.lexsort((r["seq"], r["warp"], r["launch"]))
    return np.ascontiguousarray(recs_u8)[order]


def footprint(recs_u8, n_launches):
    """F2 on-GPU consumer (P:L187 (§6.1): records "can be analyzed directly on the GPU"): per launch l,
    [distinct 32 B sectors, distinct 128 B lines, records] over the addresses of the lanes of E = A & P
    of every record of launch l — the memory footprint of the launch (reading R-18). Plain definition:
    numpy.unique of the address >> 5 / >> 7 per launch."""
    out = np.zeros((n_launches, 3), dtype=np.int64)
    r = np.ascontiguousarray(recs_u8).view(RECORD_DTYPE).reshape(-1)
    for l in range(n_launches):
        rl = r[r["launch"] == l]
        E = (rl["A"] & rl["P"]).astype(np.uint64)
        act = ((E[:, None] >> np.arange(32, dtype=np.uint64)[None, :]) & np.uint64(1)) == 1
        a = rl["addr"][act]
        out[l, 0] = len(np.unique(a >> np.uint64(5)))
        out[l, 1] = len(np.unique(a >> np.uint64(7)))
        out[l, 2] = len(rl)
    return out
