"""C3 level-synchronous BFS (Rodinia-style two-kernel) CPU model — docs/EVENT_MODEL.md §3.3.

The BFS state (mask, visited, updating, cost, over) is simulated for all vertices exactly as the two
kernels update it; events are emitted for the selected warps from the state each launch sees.
"""
import numpy as np

from . import FULL, mask_of


def n_warps(n):
    return -(-n // 256) * 8


class Ptrs:
    """Device byte addresses of the BFS buffers (only used to form event addresses)."""

    def __init__(self, mask, visited, updating, cost, over, rowptr, col):
        self.mask, self.visited, self.updating, self.cost = mask, visited, updating, cost
        self.over, self.rowptr, self.col = over, rowptr, col


def _u(base, off, scale=1):
    return np.uint64(base) + (np.asarray(off, dtype=np.int64) * scale).astype(np.uint64)


def kernel1(acc, launch, warps, rowptr, col, st, ptr):
    """Expand: events of pcs 0–21 for `warps`; returns the state changes (for all vertices)."""
    n = len(rowptr) - 1
    nw = len(warps)
    lane = np.arange(32, dtype=np.int64)[None, :]
    t = warps[:, None] * 32 + lane
    full = np.full(nw, FULL)
    for pc in range(4):
        acc.add(launch, warps, pc, full, full)
    live = t < n
    acc.add(launch, warps, 4, full, mask_of(~live))                     # @P0 EXIT
    tc = np.where(live, t, 0)
    Alive = mask_of(live)
    acc.add(launch, warps, 5, Alive, Alive, _u(ptr.mask, tc))           # LDG mask[t]
    acc.add(launch, warps, 6, Alive, Alive)
    m = live & (st["mask"][tc] != 0)
    acc.add(launch, warps, 7, Alive, mask_of(live & ~m))                # @!P1 BRA
    Af = mask_of(m)
    start = np.where(m, rowptr[tc], 0).astype(np.int64)
    end = np.where(m, rowptr[np.minimum(tc + 1, n)], 0).astype(np.int64)
    acc.add(launch, warps, 8, Af, Af, _u(ptr.mask, tc))                 # STG mask[t] = 0
    acc.add(launch, warps, 9, Af, Af, _u(ptr.rowptr, tc, 4))
    acc.add(launch, warps, 10, Af, Af, _u(ptr.rowptr, tc + 1, 4))
    acc.add(launch, warps, 11, Af, Af)
    acc.add(launch, warps, 12, Af, mask_of(m & (start >= end)))         # @P2 BRA
    deg = np.where(m, end - start, 0)
    maxdeg = deg.max(axis=1)
    order = np.argsort(-maxdeg, kind="stable")
    sorted_max = maxdeg[order]
    for k in range(int(maxdeg.max()) if nw else 0):                     # loop instances, k-th
        cnt = int(np.searchsorted(-sorted_max, -k, side="left"))       # warps with maxdeg > k
        sel = order[:cnt]
        w = warps[sel]
        ak = deg[sel] > k
        e = np.where(ak, start[sel] + k, 0)
        nb = np.where(ak, col[e], 0).astype(np.int64)
        Ak = mask_of(ak)
        acc.add(launch, w, 13, Ak, Ak, _u(ptr.col, e, 4))               # LDG col[e]
        acc.add(launch, w, 14, Ak, Ak, _u(ptr.visited, nb))             # LDG visited[nb]
        acc.add(launch, w, 15, Ak, Ak)
        vis = ak & (st["visited"][nb] != 0)
        acc.add(launch, w, 16, Ak, mask_of(vis))                        # @P3 BRA
        unv = ak & ~vis
        Au = mask_of(unv)
        acc.add(launch, w, 17, Au, Au, _u(ptr.updating, nb))            # STG updating[nb] = 1
        acc.add(launch, w, 18, Ak, Ak)
        acc.add(launch, w, 19, Ak, Ak)
        acc.add(launch, w, 20, Ak, mask_of(ak & (e + 1 < end[sel])))    # @P4 BRA
    acc.add(launch, warps, 21, Alive, Alive)                            # EXIT


def kernel2(acc, launch, warps, n, level, st, ptr):
    nw = len(warps)
    lane = np.arange(32, dtype=np.int64)[None, :]
    t = warps[:, None] * 32 + lane
    full = np.full(nw, FULL)
    for pc in range(22, 26):
        acc.add(launch, warps, pc, full, full)
    live = t < n
    acc.add(launch, warps, 26, full, mask_of(~live))                    # @P0 EXIT
    tc = np.where(live, t, 0)
    Alive = mask_of(live)
    acc.add(launch, warps, 27, Alive, Alive, _u(ptr.updating, tc))
    acc.add(launch, warps, 28, Alive, Alive)
    u = live & (st["updating"][tc] != 0)
    acc.add(launch, warps, 29, Alive, mask_of(live & ~u))               # @!P1 BRA
    Au = mask_of(u)
    acc.add(launch, warps, 30, Au, Au, _u(ptr.mask, tc))
    acc.add(launch, warps, 31, Au, Au, _u(ptr.visited, tc))
    acc.add(launch, warps, 32, Au, Au, _u(ptr.cost, tc, 4))
    acc.add(launch, warps, 33, Au, Au, _u(ptr.updating, tc))
    acc.add(launch, warps, 34, Au, Au, np.full(t.shape, np.uint64(ptr.over)))
    acc.add(launch, warps, 35, Alive, Alive)


def run(acc, rowptr, col, src, ptr, first_launch=0, warps=None):
    """Whole BFS from `src`. Returns (cost int32[n], levels, launches)."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    n = len(rowptr) - 1
    if warps is None:
        warps = np.arange(n_warps(n))
    warps = np.asarray(warps, dtype=np.int64)
    st = {
        "mask": np.zeros(n, dtype=np.uint8), "visited": np.zeros(n, dtype=np.uint8),
        "updating": np.zeros(n, dtype=np.uint8), "cost": np.full(n, -1, dtype=np.int32),
    }
    st["mask"][src] = 1
    st["visited"][src] = 1
    st["cost"][src] = 0
    level, launch = 0, first_launch
    while True:
        st["updating"][:] = 0
        kernel1(acc, launch, warps, rowptr, col, st, ptr)
        # state change of kernel 1 (all vertices): frontier mask cleared, unvisited neighbours marked
        front = np.nonzero(st["mask"])[0]
        st["mask"][front] = 0
        deg = rowptr[front + 1] - rowptr[front]
        nbrs = col[np.repeat(rowptr[front], deg) + (np.arange(deg.sum()) - np.repeat(np.cumsum(deg) - deg, deg))]
        nbrs = nbrs[st["visited"][nbrs] == 0]
        st["updating"][nbrs] = 1
        launch += 1
        kernel2(acc, launch, warps, n, level, st, ptr)
        upd = np.nonzero(st["updating"])[0]
        st["mask"][upd] = 1
        st["visited"][upd] = 1
        st["cost"][upd] = level + 1
        st["updating"][upd] = 0
        over = len(upd) > 0
        launch += 1
        level += 1
        if not over:
            break
    return st["cost"], level, launch - first_launch
