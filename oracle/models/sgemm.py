"""C2 naive SGEMM CPU model (row-fastest "strided" mapping) — docs/EVENT_MODEL.md §3.2."""
import numpy as np

from . import FULL, mask_of, warp_geometry_2d


def grid(M, N):
    return -(-M // 32), -(-N // 8)


def n_warps(M, N):
    gx, gy = grid(M, N)
    return gx * gy * 8


def run(acc, M, N, K, A_ptr, B_ptr, C_ptr, launch=0, warps=None):
    """Events of one launch of C = A·B (A: M×K, B: K×N, C: M×N, fp32 row-major at byte addresses)."""
    assert K >= 1
    gx, gy = grid(M, N)
    if warps is None:
        warps = np.arange(gx * gy * 8)
    warps = np.asarray(warps, dtype=np.int64)
    nw = len(warps)
    cx, cy, ty = warp_geometry_2d(warps, gx)
    lane = np.arange(32, dtype=np.int64)[None, :]
    row = cx[:, None] * 32 + lane                        # pc4
    col = np.broadcast_to((cy * 8 + ty)[:, None], row.shape)  # pc5 (warp-uniform)
    full = np.full(nw, FULL)
    for pc in range(7):                                  # S2R x4, IMAD, IMAD, ISETP
        acc.add(launch, warps, pc, full, full)
    p0 = (row >= M) | (col >= N)
    acc.add(launch, warps, 7, full, mask_of(p0))         # @P0 EXIT
    live = mask_of(~p0)
    acc.add(launch, warps, 8, live, live)                # MOV acc
    acc.add(launch, warps, 9, live, live)                # MOV k
    u = lambda base, off: np.uint64(base) + (off * 4).astype(np.uint64)
    for k in range(K):                                   # BB2, instance k
        acc.add(launch, warps, 10, live, live, u(A_ptr, row * K + k))
        acc.add(launch, warps, 11, live, live, u(B_ptr, k * N + col))
        acc.add(launch, warps, 12, live, live)           # FFMA
        acc.add(launch, warps, 13, live, live)           # IADD k
        acc.add(launch, warps, 14, live, live)           # ISETP k+1 < K
        p1 = live if k + 1 < K else np.zeros(nw, dtype=np.uint32)
        acc.add(launch, warps, 15, live, p1)             # @P1 BRA
    acc.add(launch, warps, 16, live, live, u(C_ptr, row * N + col))
    acc.add(launch, warps, 17, live, live)               # EXIT
