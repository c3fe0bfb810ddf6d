"""F4 instruction emulation (WFFT32) CPU model — docs/EVENT_MODEL.md §3.6; paper §6.3.

Two things are modelled, both TEST INFRASTRUCTURE (see oracle/__init__.py):
  * `dft32(x)`: what WFFT32 computes, written as its definition X[k] = Σ_n x[n]·exp(−2πi·n·k/32) in
    complex128 (a matrix product with the DFT matrix is the only library step);
  * `run(...)`: the warp-level events of one launch of either program (WFFT_EMU: the kernel that uses the
    proxy instruction, Listing 10 analogue; WFFT_SW: the transform written in CUDA), which depend only on
    n_fft and the grid (control flow does not depend on the data).
"""
import numpy as np

from . import FULL

EMU, SW = 0, 1
N = 32


def dft32(x):
    """x: complex [..., 32] -> X[..., k] = Σ_n x[..., n] exp(−2πi n k / 32), complex128 (§3.6)."""
    n = np.arange(N)
    F = np.exp(-2j * np.pi * np.outer(n, n) / N)        # F[k, n]; symmetric
    return np.asarray(x, dtype=np.complex128) @ F.T


def brev5(l):
    """5-bit bit reversal of lane ids."""
    l = np.asarray(l, dtype=np.int64)
    r = np.zeros_like(l)
    for b in range(5):
        r |= ((l >> b) & 1) << (4 - b)
    return r


def n_warps(ctas):
    return 8 * ctas


def transforms_per_warp(n_fft, ctas):
    """k_w = number of transforms warp w computes (f = w, w + W, ... < n_fft)."""
    W = n_warps(ctas)
    w = np.arange(W, dtype=np.int64)
    return np.maximum(0, -(-(n_fft - w) // W))


def run(acc, variant, n_fft, ctas, x_ptr, X_ptr, launch=0, warps=None):
    """Events of one launch of program WFFT_EMU (variant EMU) or WFFT_SW (variant SW), §3.6."""
    if n_fft == 0:                                        # nothing is launched (§3.6)
        return
    W = n_warps(ctas)
    if warps is None:
        warps = np.arange(W)
    warps = np.asarray(warps, dtype=np.int64)
    nw = len(warps)
    full = np.full(nw, FULL)
    none = np.zeros(nw, dtype=np.uint32)
    lane = np.arange(32, dtype=np.int64)
    for pc in range(4):                                   # S2R, S2R, IMAD, ISETP
        acc.add(launch, warps, pc, full, full)
    p0 = warps >= n_fft                                   # warp-uniform guard
    acc.add(launch, warps, 4, full, np.where(p0, FULL, 0).astype(np.uint32))   # @P0 EXIT
    live = warps[~p0]
    if len(live) == 0:
        return
    lf = np.full(len(live), FULL)
    if variant == SW:
        for pc in range(5, 39):                           # twiddle setup, BREV, SHF
            acc.add(launch, live, pc, lf, lf)
        lo, st_pc, ld_pc, bra_pc, exit_pc = 39, 78, 40, 81, 82
        st_lane = brev5(lane)
    else:
        lo, st_pc, ld_pc, bra_pc, exit_pc = 5, 9, 6, 12, 13
        st_lane = lane
    f, ws = live.copy(), live.copy()
    while len(f):                                          # loop instance: warps with f < n_fft
        A = np.full(len(f), FULL)
        more = f + W < n_fft
        for pc in range(lo, bra_pc + 1):
            addr = None
            if pc == ld_pc:
                addr = (np.uint64(x_ptr) + (256 * f[:, None] + 8 * lane[None, :]).astype(np.uint64))
            elif pc == st_pc:
                addr = (np.uint64(X_ptr) + (256 * f[:, None] + 8 * st_lane[None, :]).astype(np.uint64))
            P = np.where(more, FULL, 0).astype(np.uint32) if pc == bra_pc else A
            acc.add(launch, ws, pc, A, P, addr)
        f, ws = f[more] + W, ws[more]
    acc.add(launch, live, exit_pc, lf, lf)                # EXIT after the loop
