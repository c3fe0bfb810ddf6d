"""C5 event generator — docs/EVENT_MODEL.md §3.5, written out step by step."""
from __future__ import annotations

import numpy as np

from .mix import R, SEED
from . import programs

M40 = np.uint64((1 << 40) - 1)


def events(first: int, n: int, prog=None, seed: int = SEED):
    """Events first .. first+n-1 as (pc, warp, A, P, addr[n, 32] uint64 (0 for non-memory pcs))."""
    if prog is None:
        prog = programs.replay()
    i = np.arange(first, first + n, dtype=np.uint64)
    pc = (R(i, 0, seed) % np.uint64(4096)).astype(np.int64)
    warp = (R(i, 1, seed) % np.uint64(1 << 20)).astype(np.int64)
    r2, r3 = R(i, 2, seed), R(i, 3, seed)
    A = np.where(r2 % np.uint64(4) != 0, np.uint64(0xFFFFFFFF), r3 & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    A = np.where(A == 0, np.uint32(1), A)
    r4, r5 = R(i, 4, seed), R(i, 5, seed)
    P = np.where(r4 % np.uint64(8) < 6, np.uint64(0xFFFFFFFF), r5 & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    addr = np.zeros((n, 32), dtype=np.uint64)
    mem = programs.is_mem(prog)[pc]
    if mem.any():
        mi = i[mem]
        wd = prog["width"][pc[mem]].astype(np.uint64)[:, None]
        pat = (R(mi, 6, seed) % np.uint64(6))[:, None]
        base = ((R(mi, 7, seed) & M40) & ~np.uint64(127))[:, None]
        s = R(mi, 8, seed)[:, None]
        lane = np.arange(32, dtype=np.uint64)[None, :]
        r = np.stack([R(mi, 64 + l, seed) for l in range(32)], axis=1)
        with np.errstate(over="ignore"):
            a0 = base + lane * wd
            a1 = base + lane * (wd << (s % np.uint64(10)))
            a2 = np.broadcast_to(base, r.shape)
            a3 = base + (r % (np.uint64(4096) // wd)) * wd
            a4 = (r & M40) & ~(wd - np.uint64(1))
            a5 = base + (lane ^ (s & np.uint64(31))) * wd
        a = np.select([pat == 0, pat == 1, pat == 2, pat == 3, pat == 4],
                      [a0, a1, a2, a3, a4], a5)
        addr[mem] = a
    return pc, warp, A, P, addr


def replay(acc, first: int, n: int, chunk: int = 1 << 16, seed: int = SEED):
    """Apply §2 items 1–4 to events [first, first+n) (acc built on programs.replay(seed))."""
    for c0 in range(first, first + n, chunk):
        m = min(chunk, first + n - c0)
        pc, warp, A, P, addr = events(c0, m, acc.prog, seed)
        acc.add(0, warp, pc, A, P, addr)


def header_bytes(pc, warp, A, P):
    """The replay stream's 16-byte headers {u32 pc, u32 warp, u32 A, u32 P}."""
    h = np.zeros((len(pc), 4), dtype="<u4")
    h[:, 0], h[:, 1], h[:, 2], h[:, 3] = pc, warp, A, P
    return h
