"""C1 vectorAdd CPU model — docs/EVENT_MODEL.md §3.1."""
import numpy as np

from . import FULL, mask_of


def n_warps(N):
    return -(-N // 256) * 8


def run(acc, N, a, b, c, launch=0, warps=None):
    """Emit the events of one launch of vectorAdd over N elements (buffers at byte addresses a, b, c)."""
    if warps is None:
        warps = np.arange(n_warps(N))
    warps = np.asarray(warps, dtype=np.int64)
    nw = len(warps)
    lane = np.arange(32, dtype=np.int64)[None, :]
    i = warps[:, None] * 32 + lane               # ctaid.x*256 + tid.x, 8 warps per CTA
    full = np.full(nw, FULL)
    for pc in range(4):                          # S2R, S2R, IMAD, ISETP: every lane
        acc.add(launch, warps, pc, full, full)
    p0 = mask_of(i >= N)
    acc.add(launch, warps, 4, full, p0)          # @P0 EXIT
    A = mask_of(i < N)                           # lanes that executed EXIT are gone
    ua = lambda base: (np.uint64(base) + (i * 4).astype(np.uint64))
    for pc in range(5, 13):
        addr = {7: ua(a), 8: ua(b), 11: ua(c)}.get(pc)
        acc.add(launch, warps, pc, A, A, addr)
