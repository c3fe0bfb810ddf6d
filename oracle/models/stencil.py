"""C4 5-point Jacobi stencil CPU model — docs/EVENT_MODEL.md §3.4."""
import numpy as np

from . import FULL, mask_of, warp_geometry_2d


def grid(n):
    return -(-n // 32), -(-n // 8)


def n_warps(n):
    gx, gy = grid(n)
    return gx * gy * 8


def run(acc, n, in_ptr, out_ptr, launch=0, warps=None):
    """Events of one launch reading grid `in_ptr` and writing `out_ptr` (n×n fp32, row-major)."""
    gx, gy = grid(n)
    if warps is None:
        warps = np.arange(gx * gy * 8)
    warps = np.asarray(warps, dtype=np.int64)
    nw = len(warps)
    cx, cy, ty = warp_geometry_2d(warps, gx)
    lane = np.arange(32, dtype=np.int64)[None, :]
    j = cx[:, None] * 32 + lane
    i = np.broadcast_to((cy * 8 + ty)[:, None], j.shape)
    full = np.full(nw, FULL)
    for pc in range(7):                                   # S2R x4, IMAD j, IMAD i, ISETP
        acc.add(launch, warps, pc, full, full)
    p0 = (i >= n) | (j >= n)
    acc.add(launch, warps, 7, full, mask_of(p0))          # @P0 EXIT
    live = ~p0
    A = mask_of(live)
    P1 = mask_of(live & (i > 0) & (i < n - 1) & (j > 0) & (j < n - 1))
    u = lambda off: np.uint64(in_ptr) + (off * 4).astype(np.uint64)
    acc.add(launch, warps, 8, A, A)                       # ISETP P1
    acc.add(launch, warps, 9, A, A, u(i * n + j))         # center
    acc.add(launch, warps, 10, A, P1, u((i - 1) * n + j))  # @P1 up
    acc.add(launch, warps, 11, A, P1, u((i + 1) * n + j))  # @P1 down
    acc.add(launch, warps, 12, A, P1, u(i * n + j - 1))    # @P1 left
    acc.add(launch, warps, 13, A, P1, u(i * n + j + 1))    # @P1 right
    for pc in (14, 15, 16, 17):                           # @P1 FADD x3, FMUL
        acc.add(launch, warps, pc, A, P1)
    acc.add(launch, warps, 18, A, A)                      # SEL
    acc.add(launch, warps, 19, A, A, np.uint64(out_ptr) + ((i * n + j) * 4).astype(np.uint64))
    acc.add(launch, warps, 20, A, A)                      # EXIT


def run_iterations(acc, n, buf0, buf1, iters, first_launch=0, warps=None):
    """Iteration `it` reads buffer it%2 and writes buffer (it+1)%2 (launch id first_launch + it)."""
    bufs = (buf0, buf1)
    for it in range(iters):
        run(acc, n, bufs[it % 2], bufs[(it + 1) % 2], launch=first_launch + it, warps=warps)


def jacobi_reference(x, iters):
    """Plain fp32 Jacobi on a numpy grid (for checking the kernel's output values)."""
    x = x.astype(np.float32).copy()
    for _ in range(iters):
        y = x.copy()
        y[1:-1, 1:-1] = np.float32(0.25) * (((x[:-2, 1:-1] + x[2:, 1:-1]) + x[1:-1, :-2]) + x[1:-1, 2:])
        x = y
    return x
