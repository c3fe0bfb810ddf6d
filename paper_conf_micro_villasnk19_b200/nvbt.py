"""Thin ctypes binding of libnvbt.so (include/nvbt.h, include/nvbt_workloads.h).

Argument marshalling only: every step of the hot path runs in the library's CUDA kernels. PyTorch
supplies device memory (workspace, streams of events, workload buffers), pinned host memory (the
trace ring) and streams. The library must be built (`python -m paper_conf_micro_villasnk19_b200.build`
or `__graft_entry__.build()`); there is no fallback — a missing library raises at import.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# NVBT_LIB selects another build of the library (tests load libnvbt_debug.so, the converged-hook check)
LIB_PATH = os.environ.get("NVBT_LIB") or os.path.join(_HERE, "libnvbt.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libnvbt.so not built at {LIB_PATH}; run __graft_entry__.build()")
_lib = C.CDLL(LIB_PATH)

ABI_VERSION = 1
OK, EINVAL, ESTATE, ENOMEM, ECUDA, ETIMEDOUT, EVERSION = 0, -1, -2, -3, -4, -5, -6
COUNT, OPHIST, BB, MEMDIV, PER_WARP, TRACE = 1, 2, 4, 8, 16, 32
TOOL_NONE, TOOL_COUNT, TOOL_BBCOUNT, TOOL_MEMDIV, TOOL_TRACE, TOOL_EMU = 0, 1, 2, 4, 8, 16
W_VECTORADD, W_SGEMM, W_BFS, W_STENCIL, W_REPLAY, W_WFFT_EMU, W_WFFT_SW = 1, 2, 3, 4, 5, 6, 7
WFFT_PROXY, WFFT_SOFTWARE = 0, 1
RECORD_BYTES = 288
COMPACT_RECORD_BYTES = 176
COMPACT128_RECORD_BYTES = 128


class InstrDesc(C.Structure):
    _fields_ = [("opcode", C.c_uint16), ("kind", C.c_uint8), ("width", C.c_uint8), ("bb", C.c_uint32),
                ("is_leader", C.c_uint8), ("guarded", C.c_uint8), ("pad", C.c_uint16)]


class Config(C.Structure):
    _fields_ = [("version", C.c_uint32), ("device", C.c_int32), ("stream", C.c_void_p),
                ("prog", C.POINTER(InstrDesc)), ("n_pcs", C.c_uint32), ("n_opcodes", C.c_uint32),
                ("n_bbs", C.c_uint32), ("n_warps", C.c_uint32), ("flags", C.c_uint32),
                ("d_workspace", C.c_void_p), ("workspace_bytes", C.c_size_t)]


class Counts(C.Structure):
    _fields_ = [("thread_issued", C.c_uint64), ("thread_exec", C.c_uint64),
                ("warp_issued", C.c_uint64), ("warp_exec", C.c_uint64)]


class MemDiv(C.Structure):
    _fields_ = [("accesses", C.c_uint64), ("sectors", C.c_uint64), ("lines", C.c_uint64)]


class MemDivTotal(C.Structure):
    _fields_ = [("sum", MemDiv), ("hist_sectors", C.c_uint64 * 33), ("hist_lines", C.c_uint64 * 33)]


class Digest(C.Structure):
    _fields_ = [("n_rec", C.c_uint64), ("d1", C.c_uint64), ("d2", C.c_uint64)]


class CopySink(C.Structure):
    _fields_ = [("dst", C.c_void_p), ("capacity", C.c_uint64), ("n", C.c_uint64)]


class DevState(C.Structure):
    """nvbt_dev_state (include/nvbt.h): the POD an external instrumented kernel receives by value."""
    _fields_ = [("version", C.c_uint32), ("tools", C.c_uint32), ("site", C.c_void_p), ("mem", C.c_void_p),
                ("hist", C.c_void_p), ("per_warp", C.c_void_p), ("stripe_words", C.c_uint64),
                ("stripes", C.c_uint32), ("n_pcs", C.c_uint32), ("n_warps", C.c_uint32), ("launch", C.c_uint32)]


DRAIN_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_uint64, C.c_void_p)

_P = C.c_void_p
_sigs = {
    "nvbt_abi_version": ([], C.c_int),
    "nvbt_last_error": ([], C.c_char_p),
    "nvbt_workspace_size": ([C.POINTER(Config), C.POINTER(C.c_size_t)], C.c_int),
    "nvbt_init": ([C.POINTER(Config), C.POINTER(_P)], C.c_int),
    "nvbt_reset": ([_P], C.c_int),
    "nvbt_fini": ([_P], C.c_int),
    "nvbt_accum_view": ([_P, C.POINTER(_P), C.POINTER(C.c_size_t)], C.c_int),
    "nvbt_accum_axpy": ([_P, _P, C.c_size_t, C.c_int64], C.c_int),
    "nvbt_count": ([_P, C.POINTER(Counts), _P, _P], C.c_int),
    "nvbt_opcode_hist": ([_P, _P, _P, C.c_uint32], C.c_int),
    "nvbt_bb_count": ([_P, _P, C.c_uint32], C.c_int),
    "nvbt_mem_divergence": ([_P, _P, C.c_uint32, C.POINTER(MemDivTotal)], C.c_int),
    "nvbt_channel_bytes": ([C.c_uint32, C.c_uint64, C.c_int], C.c_size_t),
    "nvbt_channel_open": ([_P, _P, C.c_size_t, C.c_uint32, C.POINTER(_P)], C.c_int),
    "nvbt_channel_drain": ([_P, _P, _P, C.c_int64, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_channel_close": ([_P], C.c_int),
    "nvbt_channel_dropped": ([_P, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_digest_records": ([_P, C.c_uint64, C.POINTER(Digest)], C.c_int),
    "nvbt_decode_compact": ([_P, C.c_uint64, _P, C.c_uint64, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_decode_slots": ([_P, C.c_uint64, C.c_uint32, _P, C.c_uint64, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_trace_footprint": ([_P, _P, C.c_uint64, C.c_uint32, C.c_uint32, _P, _P], C.c_int),
    "nvbt_gen_events": ([_P, C.c_uint64, C.c_uint64, C.c_uint64, _P, _P], C.c_int),
    "nvbt_replay": ([_P, _P, _P, C.c_uint64], C.c_int),
    "nvbt_replay_errors": ([_P, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_replay_scratch_size": ([_P, C.c_uint64, C.POINTER(C.c_size_t)], C.c_int),
    "nvbt_replay_staged": ([_P, _P, _P, C.c_uint64, _P, C.c_size_t], C.c_int),
    "nvbt_launch_count": ([_P, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_program": ([C.c_int, _P, C.c_uint32, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32),
                      C.POINTER(C.c_uint32)], C.c_int),
    "nvbt_workload_warps": ([C.c_int, C.POINTER(C.c_int64), C.c_uint32, C.POINTER(C.c_uint64)], C.c_int),
    "nvbt_vectoradd": ([_P, _P, C.c_uint32, _P, _P, _P, C.c_int32], C.c_int),
    "nvbt_sgemm": ([_P, _P, C.c_uint32, _P, _P, _P, C.c_int32, C.c_int32, C.c_int32], C.c_int),
    "nvbt_bfs_level": ([_P, _P, C.c_uint32, _P, _P, C.c_int32, _P, _P, _P, _P, _P, C.c_int32], C.c_int),
    "nvbt_stencil": ([_P, _P, C.c_uint32, _P, _P, C.c_int32], C.c_int),
    "nvbt_bfs_expand": ([_P, _P, C.c_uint32, _P, _P, C.c_int32, _P, _P, _P], C.c_int),
    "nvbt_bfs_update": ([_P, _P, C.c_uint32, C.c_int32, _P, _P, _P, _P, _P, C.c_int32], C.c_int),
    "nvbt_set_partition": ([_P, C.c_uint32, C.c_uint32], C.c_int),
    "nvbt_device_state": ([_P, C.c_uint32, _P, C.c_size_t], C.c_int),
    "nvbt_wfft32": ([_P, _P, C.c_uint32, C.c_int32, _P, _P, C.c_int32, C.c_int32], C.c_int),
    "nvbt_wfft32_max_ctas": ([C.c_uint32, C.c_int32, C.c_int32, C.POINTER(C.c_int32)], C.c_int),
}
for _name, (_args, _res) in _sigs.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res
EXPORTED = tuple(_sigs) + ("nvbt_drain_digest", "nvbt_drain_copy", "nvbt_drain_discard")
_DRAIN_DIGEST = C.cast(_lib.nvbt_drain_digest, C.c_void_p).value
_DRAIN_COPY = C.cast(_lib.nvbt_drain_copy, C.c_void_p).value
_DRAIN_DISCARD = C.cast(_lib.nvbt_drain_discard, C.c_void_p).value


class NvbtError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"nvbt error {code}: {msg}")
        self.code = code


def _check(rc):
    if rc != OK:
        raise NvbtError(rc, _lib.nvbt_last_error().decode(errors="replace"))
    return rc


def _ptr(t):
    return None if t is None else C.c_void_p(t.data_ptr())


def _stream_handle(stream):
    import torch
    s = torch.cuda.current_stream() if stream is None else stream
    return s.cuda_stream


# ------------------------------------------------------------------------------------------- host-only
def nvbt_abi_version():
    return _lib.nvbt_abi_version()


def nvbt_program(workload):
    """The workload's program table as a numpy structured array + (n_opcodes, n_bbs)."""
    n, o, b = C.c_uint32(), C.c_uint32(), C.c_uint32()
    _check(_lib.nvbt_program(workload, None, 0, C.byref(n), C.byref(o), C.byref(b)))
    arr = (InstrDesc * n.value)()
    _check(_lib.nvbt_program(workload, C.cast(arr, C.c_void_p), n.value, None, None, None))
    return arr, o.value, b.value


def program_numpy(arr):
    """InstrDesc array -> dict of numpy arrays (same keys as the oracle's programs, for tests)."""
    f = lambda k: np.array([getattr(d, k) for d in arr], dtype=np.int64)
    return {k: f(k) for k in ("opcode", "kind", "width", "bb", "is_leader", "guarded")}


def nvbt_workload_warps(workload, *args):
    a = (C.c_int64 * len(args))(*args)
    n = C.c_uint64()
    _check(_lib.nvbt_workload_warps(workload, a, len(args), C.byref(n)))
    return n.value


def nvbt_workspace_size(prog_len, n_opcodes, n_bbs, flags, n_warps=0):
    cfg = Config(ABI_VERSION, 0, None, None, prog_len, n_opcodes, n_bbs, n_warps, flags, None, 0)
    b = C.c_size_t()
    _check(_lib.nvbt_workspace_size(C.byref(cfg), C.byref(b)))
    return b.value


def nvbt_decode_compact(slots_u8, record_bytes=COMPACT_RECORD_BYTES):
    """Decode a numpy uint8 [n, record_bytes] array of compact transport slots (176: EM §5.1, 128: EM §5.2)
    into EM §5 records [m, 288]."""
    sl = np.ascontiguousarray(slots_u8, dtype=np.uint8)
    out = np.zeros((sl.shape[0], RECORD_BYTES), dtype=np.uint8)
    k = C.c_uint64()
    _check(_lib.nvbt_decode_slots(sl.ctypes.data_as(C.c_void_p), sl.shape[0], record_bytes,
                                  out.ctypes.data_as(C.c_void_p), sl.shape[0], C.byref(k)))
    return out[:k.value]


def nvbt_digest_records(records_u8):
    """Host digest (EM §5) of a contiguous numpy uint8 [n, 288] array."""
    r = np.ascontiguousarray(records_u8, dtype=np.uint8)
    d = Digest()
    _check(_lib.nvbt_digest_records(r.ctypes.data_as(C.c_void_p), r.shape[0], C.byref(d)))
    return d.n_rec, d.d1, d.d2


# ------------------------------------------------------------------------------------------- context
class Ctx:
    """An nvbt context: the handle plus the torch tensors it borrows (workspace)."""

    def __init__(self, handle, workspace, prog, n_opcodes, n_bbs, n_warps, flags, device, stream):
        self.handle, self.workspace = handle, workspace
        self.n_pcs, self.n_opcodes, self.n_bbs, self.n_warps = len(prog), n_opcodes, n_bbs, n_warps
        self.flags, self.device, self.stream = flags, device, stream
        self.prog = prog
        self.channel = None

    def __del__(self):
        if getattr(self, "handle", None):
            try:
                _lib.nvbt_fini(self.handle)
            except Exception:
                pass
            self.handle = None


def nvbt_init(workload_or_prog, flags, n_warps=0, device=None, stream=None, n_opcodes=None, n_bbs=None):
    """Allocate the workspace (torch, on `device`) and initialise a context on `stream`.

    workload_or_prog: a workload id (W_*) or an InstrDesc array (then n_opcodes/n_bbs are required)."""
    import torch
    if isinstance(workload_or_prog, int):
        prog, n_opcodes, n_bbs = nvbt_program(workload_or_prog)
    else:
        prog = workload_or_prog
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    with torch.cuda.device(dev):
        sh = _stream_handle(stream)
        cfg = Config(ABI_VERSION, dev.index, C.c_void_p(sh), C.cast(prog, C.POINTER(InstrDesc)), len(prog),
                     n_opcodes, n_bbs, n_warps, flags, None, 0)
        b = C.c_size_t()
        _check(_lib.nvbt_workspace_size(C.byref(cfg), C.byref(b)))
        ws = torch.empty(b.value, dtype=torch.uint8, device=dev)
        cfg.d_workspace = C.c_void_p(ws.data_ptr())
        cfg.workspace_bytes = b.value
        h = C.c_void_p()
        _check(_lib.nvbt_init(C.byref(cfg), C.byref(h)))
    return Ctx(h, ws, prog, n_opcodes, n_bbs, n_warps, flags, dev, stream)


def nvbt_reset(ctx):
    _check(_lib.nvbt_reset(ctx.handle))


def nvbt_fini(ctx):
    if ctx.handle:
        _check(_lib.nvbt_fini(ctx.handle))
        ctx.handle = None


def nvbt_accum_view(ctx):
    """int64 torch view of the packed accumulator region (for dist.all_reduce)."""
    import torch
    p, n = C.c_void_p(), C.c_size_t()
    _check(_lib.nvbt_accum_view(ctx.handle, C.byref(p), C.byref(n)))
    off = p.value - ctx.workspace.data_ptr()
    return ctx.workspace[off:off + 8 * n.value].view(torch.int64)


def nvbt_accum_axpy(ctx, src, factor):
    """accum += factor * src (src: int64 CUDA tensor with the accumulator layout)."""
    _check(_lib.nvbt_accum_axpy(ctx.handle, C.c_void_p(src.data_ptr()), src.numel(), int(factor)))


def nvbt_count(ctx, per_warp=False):
    c = Counts()
    pwt = pww = None
    if per_warp:
        pwt = np.zeros(ctx.n_warps, dtype=np.uint64)
        pww = np.zeros(ctx.n_warps, dtype=np.uint64)
    _check(_lib.nvbt_count(ctx.handle, C.byref(c), None if pwt is None else pwt.ctypes.data_as(C.c_void_p),
                           None if pww is None else pww.ctypes.data_as(C.c_void_p)))
    out = np.array([c.thread_issued, c.thread_exec, c.warp_issued, c.warp_exec], dtype=np.uint64)
    return (out, pwt, pww) if per_warp else out


def nvbt_opcode_hist(ctx):
    t = np.zeros(ctx.n_opcodes, dtype=np.uint64)
    w = np.zeros(ctx.n_opcodes, dtype=np.uint64)
    _check(_lib.nvbt_opcode_hist(ctx.handle, t.ctypes.data_as(C.c_void_p), w.ctypes.data_as(C.c_void_p),
                                 ctx.n_opcodes))
    return t, w


def nvbt_bb_count(ctx):
    """[n_bbs, 4]: entries_warp, entries_thread, instrs_warp, instrs_thread."""
    out = np.zeros((ctx.n_bbs, 4), dtype=np.uint64)
    _check(_lib.nvbt_bb_count(ctx.handle, out.ctypes.data_as(C.c_void_p), ctx.n_bbs))
    return out


def nvbt_mem_divergence(ctx):
    """(per_pc [n_pcs, 3] n/ΣS/ΣL, total (3,), hist_sectors (33,), hist_lines (33,))."""
    per = np.zeros((ctx.n_pcs, 3), dtype=np.uint64)
    tot = MemDivTotal()
    _check(_lib.nvbt_mem_divergence(ctx.handle, per.ctypes.data_as(C.c_void_p), ctx.n_pcs, C.byref(tot)))
    s = np.array([tot.sum.accesses, tot.sum.sectors, tot.sum.lines], dtype=np.uint64)
    return per, s, np.array(tot.hist_sectors[:], dtype=np.uint64), np.array(tot.hist_lines[:], dtype=np.uint64)


def nvbt_launch_count(ctx):
    n = C.c_uint64()
    _check(_lib.nvbt_launch_count(ctx.handle, C.byref(n)))
    return n.value


# ------------------------------------------------------------------------------------------- channel
class Channel:
    def __init__(self, handle, ctx, ring):
        self.handle, self.ctx, self.ring = handle, ctx, ring


def _record_bytes(compact):
    """compact: False (288 B records), True or 176 (176 B slots, EM §5.1), 128 (128 B slots, EM §5.2)."""
    if compact is False or compact is None or compact == 0:
        return RECORD_BYTES
    if compact is True or compact == COMPACT_RECORD_BYTES:
        return COMPACT_RECORD_BYTES
    if compact == COMPACT128_RECORD_BYTES:
        return COMPACT128_RECORD_BYTES
    raise ValueError(f"compact={compact!r}: use False, True / 176 or 128")


def nvbt_channel_slot_bytes(compact=False):
    """Ring stride of one transport slot: 288, 192 (176 B slots, EM §5.1, padded) or 128 (EM §5.2)."""
    rb = _record_bytes(compact)
    return 192 if rb == COMPACT_RECORD_BYTES else rb


def nvbt_channel_bytes(slots, compact=False, on_device=False):
    """Ring size (bytes) that holds `slots` slots: header + slots * (slot stride + 4-byte tag) for host rings."""
    return int(_lib.nvbt_channel_bytes(_record_bytes(compact), slots, 1 if on_device else 0))


def nvbt_channel_open(ctx, ring, compact=False):
    """ring: pinned uint8 torch tensor (torch.empty(..., pin_memory=True)), or a CUDA uint8 tensor for an
    on-GPU channel (F2); compact: False (288 B records), True / 176 (base + 32-bit deltas, EM §5.1) or 128
    (one 128 B line per record with 16-bit deltas, EM §5.2)."""
    h = C.c_void_p()
    _check(_lib.nvbt_channel_open(ctx.handle, C.c_void_p(ring.data_ptr()), ring.numel(), _record_bytes(compact),
                                  C.byref(h)))
    ch = Channel(h, ctx, ring)
    ctx.channel = ch
    return ch


def nvbt_channel_close(ch):
    if ch.handle:
        _check(_lib.nvbt_channel_close(ch.handle))
        ch.handle = None
        ch.ctx.channel = None


def nvbt_trace_footprint(ch, n_launches, table_slots=1 << 10, scratch=None, timing=None, first_launch=0):
    """F2: per-launch (distinct sectors, distinct lines, records) of a device-memory channel [n, 3]
    for launch ids first_launch .. first_launch + n_launches - 1.
    table_slots: power of two above the distinct (launch, 1 MB region) pairs."""
    import torch
    if scratch is None:
        scratch = torch.empty(513 * table_slots + 3 * n_launches + 1, dtype=torch.int64, device=ch.ctx.device)
    out = np.zeros((n_launches, 3), dtype=np.uint64)
    ms = C.c_float(0.0)
    _check(_lib.nvbt_trace_footprint(ch.handle, C.c_void_p(scratch.data_ptr()), table_slots, first_launch, n_launches,
                                     out.ctypes.data_as(C.c_void_p), C.byref(ms) if timing is not None else None))
    if timing is not None:
        timing.append(ms.value / 1e3)   # consumer kernel device seconds
    return out


def nvbt_channel_dropped(ch):
    n = C.c_uint64()
    _check(_lib.nvbt_channel_dropped(ch.handle, C.byref(n)))
    return n.value


def nvbt_channel_drain_digest(ch, timeout_us=-1, digest=None):
    """Drain with the built-in digest callback; returns (n_rec, d1, d2) accumulated into `digest`."""
    d = Digest() if digest is None else digest
    n = C.c_uint64()
    _check(_lib.nvbt_channel_drain(ch.handle, C.c_void_p(_DRAIN_DIGEST), C.byref(d), timeout_us, C.byref(n)))
    return d


def nvbt_channel_drain_discard(ch, timeout_us=-1):
    """Drain with the built-in discard callback (transport only); returns the number of records."""
    cnt = C.c_uint64()
    n = C.c_uint64()
    _check(_lib.nvbt_channel_drain(ch.handle, C.c_void_p(_DRAIN_DISCARD), C.byref(cnt), timeout_us, C.byref(n)))
    return n.value


def nvbt_channel_drain_copy(ch, dst, timeout_us=-1):
    """Drain into a numpy uint8 [capacity, 288] array; returns the number of records copied."""
    s = CopySink(dst.ctypes.data, dst.shape[0], 0)
    n = C.c_uint64()
    _check(_lib.nvbt_channel_drain(ch.handle, C.c_void_p(_DRAIN_COPY), C.byref(s), timeout_us, C.byref(n)))
    return s.n


def nvbt_channel_drain(ch, fn, timeout_us=-1):
    """Drain with a Python callback fn(records_u8_numpy_view) -> None (slow; small tests only)."""
    def _cb(ptr, n, user):
        buf = (C.c_uint8 * (n * RECORD_BYTES)).from_address(ptr)
        fn(np.frombuffer(buf, dtype=np.uint8).reshape(n, RECORD_BYTES))
        return 0
    cb = DRAIN_FN(_cb)
    n = C.c_uint64()
    _check(_lib.nvbt_channel_drain(ch.handle, C.cast(cb, C.c_void_p), None, timeout_us, C.byref(n)))
    return n.value


# ------------------------------------------------------------------------------------------- replay
def nvbt_gen_events(ctx, seed, first, n, hdr, addr):
    _check(_lib.nvbt_gen_events(ctx.handle, seed, first, n, _ptr(hdr), _ptr(addr)))


def nvbt_replay(ctx, hdr, addr, n):
    _check(_lib.nvbt_replay(ctx.handle, _ptr(hdr), _ptr(addr), n))


def nvbt_replay_scratch_size(ctx, max_events_per_block):
    b = C.c_size_t()
    _check(_lib.nvbt_replay_scratch_size(ctx.handle, max_events_per_block, C.byref(b)))
    return b.value


def nvbt_replay_staged(ctx, hdr, addr, n, scratch):
    """scratch: a device tensor (uint8) of at least nvbt_replay_scratch_size(ctx, 1) bytes, or None."""
    nbytes = 0 if scratch is None else scratch.numel() * scratch.element_size()
    _check(_lib.nvbt_replay_staged(ctx.handle, _ptr(hdr), _ptr(addr), n, None if scratch is None else _ptr(scratch),
                                   nbytes))


def nvbt_replay_errors(ctx):
    n = C.c_uint64()
    _check(_lib.nvbt_replay_errors(ctx.handle, C.byref(n)))
    return n.value


# ------------------------------------------------------------------------------------------- workloads
def _h(ctx):
    return None if ctx is None else ctx.handle


def _s(ctx, stream):
    if ctx is not None:
        return None
    return C.c_void_p(_stream_handle(stream))


def nvbt_vectoradd(ctx, tools, a, b, c, N, stream=None):
    _check(_lib.nvbt_vectoradd(_h(ctx), _s(ctx, stream), tools, _ptr(a), _ptr(b), _ptr(c), N))


def nvbt_sgemm(ctx, tools, A, B, Cm, M, N, K, stream=None):
    _check(_lib.nvbt_sgemm(_h(ctx), _s(ctx, stream), tools, _ptr(A), _ptr(B), _ptr(Cm), M, N, K))


def nvbt_bfs_level(ctx, tools, rowptr, col, n, mask, visited, updating, cost, over, level, stream=None):
    _check(_lib.nvbt_bfs_level(_h(ctx), _s(ctx, stream), tools, _ptr(rowptr), _ptr(col), n, _ptr(mask),
                               _ptr(visited), _ptr(updating), _ptr(cost), _ptr(over), level))


def nvbt_stencil(ctx, tools, inp, out, n, stream=None):
    _check(_lib.nvbt_stencil(_h(ctx), _s(ctx, stream), tools, _ptr(inp), _ptr(out), n))


def nvbt_wfft32(ctx, tools, variant, x, X, n_fft, ctas, stream=None):
    """F4 (EM §3.6): n_fft 32-point FFTs of x (complex64 CUDA tensor [n_fft, 32]) into X."""
    _check(_lib.nvbt_wfft32(_h(ctx), _s(ctx, stream), tools, variant, _ptr(x), _ptr(X), n_fft, ctas))


def nvbt_wfft32_max_ctas(tools, variant, device=0):
    """Grid of one resident wave for the kernel (tools, variant) selects."""
    n = C.c_int32()
    _check(_lib.nvbt_wfft32_max_ctas(tools, variant, device, C.byref(n)))
    return n.value


def nvbt_bfs_expand(ctx, tools, rowptr, col, n, mask, visited, updating, stream=None):
    _check(_lib.nvbt_bfs_expand(_h(ctx), _s(ctx, stream), tools, _ptr(rowptr), _ptr(col), n, _ptr(mask),
                                _ptr(visited), _ptr(updating)))


def nvbt_bfs_update(ctx, tools, n, mask, visited, updating, cost, over, level, stream=None):
    _check(_lib.nvbt_bfs_update(_h(ctx), _s(ctx, stream), tools, n, _ptr(mask), _ptr(visited), _ptr(updating),
                                _ptr(cost), _ptr(over), level))


def nvbt_set_partition(ctx, rank, world):
    """Later workload launches through ctx run only `rank`'s share of their CTA grid."""
    _check(_lib.nvbt_set_partition(ctx.handle, rank, world))
    ctx.partition = (rank, world)


def nvbt_device_state(ctx, tools):
    """The nvbt_dev_state POD for one launch of an external kernel instrumented with include/nvbt_dev.cuh
    (tools: COUNT or BBCOUNT, optionally MEMDIV). Pass C.byref(result) to the kernel's launcher."""
    st = DevState()
    _check(_lib.nvbt_device_state(ctx.handle, tools, C.byref(st), C.sizeof(DevState)))
    return st
