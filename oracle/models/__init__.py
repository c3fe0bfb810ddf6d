"""CPU models of the synthetic workloads (docs/EVENT_MODEL.md §3.1–3.4).

Each model walks its kernel's program in program order, one dynamic instance at a time, for a set of
warps at once (numpy arrays over warps × 32 lanes), and hands each instance's events to an
`oracle.events.Accumulator`. Active masks follow the O-2 model (EVENT_MODEL §1): exited lanes leave A,
divergent paths get the lanes that take them, loop instances are aligned by iteration index.
"""
import numpy as np

FULL = np.uint32(0xFFFFFFFF)


def mask_of(bits):
    """bool [n, 32] -> uint32 [n] with bit l = bits[:, l]."""
    b = np.asarray(bits, dtype=np.uint64)
    return (b << np.arange(32, dtype=np.uint64)[None, :]).sum(axis=1).astype(np.uint32)


def warp_geometry_2d(warps, gx, bdx=32, bdy=8):
    """For CTA (32, 8) kernels: global warp id -> (ctaid.x, ctaid.y, tid.y) (lane = tid.x)."""
    warps = np.asarray(warps, dtype=np.int64)
    wpc = bdx * bdy // 32
    cta = warps // wpc
    return cta % gx, cta // gx, warps % wpc
