"""ctypes front end of the multithreaded C oracle (oracle/c/nvbt_oracle.c) — TEST INFRASTRUCTURE ONLY.

The C oracle applies docs/EVENT_MODEL.md event by event, like oracle/events.py + oracle/models, on all
host cores; it exists so that BASELINE.json's full-size configs can be checked element by element. It is
pinned against the numpy oracle and against closed forms in tests/test_oracle_c.py. Results come back in
the numpy oracle's dictionary form (`Accumulator.result()` keys), so either side compares the same way.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference) may use it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(_HERE, "c", "nvbt_oracle.c")
LIB = os.path.join(_HERE, "c", "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-fPIC", "-shared", "-pthread", "-Wall", "-Wno-unused-function"]

_lib = None


def build(force: bool = False) -> str:
    """gcc -O2 -shared the oracle in-tree (a plain C compile; no -march, no fast-math)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".{os.getpid()}.tmp"
        r = subprocess.run(["gcc", *CFLAGS, SRC, "-o", tmp], capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"oracle build failed:\n{r.stdout}{r.stderr}")
        os.replace(tmp, LIB)
    return LIB


class _Prog(C.Structure):
    _fields_ = [("n_pcs", C.c_uint32), ("n_ops", C.c_uint32), ("n_bbs", C.c_uint32),
                ("opcode", C.c_void_p), ("kind", C.c_void_p), ("width", C.c_void_p), ("bb", C.c_void_p),
                ("is_leader", C.c_void_p)]


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        P, u32, u64, i64, vp, ci = C.POINTER(_Prog), C.c_uint32, C.c_uint64, C.c_int64, C.c_void_p, C.c_int
        sig = {
            "orc_result_words": ([u32, u32, u32, u64], C.c_size_t),
            "orc_mix64": ([u64], u64),
            "orc_sectors_lines": ([vp, u32, vp, vp], None),
            "orc_events": ([P, u32, u64, vp, vp, vp, vp, vp, u64, ci, vp], ci),
            "orc_vectoradd": ([P, i64, u64, u64, u64, u32, u64, u64, ci, u64, ci, vp], ci),
            "orc_sgemm": ([P, i64, i64, i64, u64, u64, u64, u32, u64, u64, ci, u64, ci, vp], ci),
            "orc_stencil": ([P, i64, u64, u64, i64, u32, u64, u64, ci, ci, vp], ci),
            "orc_bfs": ([P, i64, vp, vp, i64, vp, u32, u64, u64, ci, u64, ci, vp, vp, vp], ci),
            "orc_gen_events": ([P, u64, u64, u64, vp, vp], None),
            "orc_replay": ([P, u64, u64, u64, ci, vp], ci),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes, f.restype = args, res
        _lib = L
    return _lib


def host_threads() -> int:
    """T = the host cores this process may run on (SURVEY §8(c).1 timing protocol)."""
    return len(os.sched_getaffinity(0))


class Prog:
    """A program table (oracle/programs.py dict) marshalled for the C side."""

    def __init__(self, prog):
        self.prog = prog
        self._cols = {k: np.ascontiguousarray(prog[k], dtype=np.int32) for k in
                      ("opcode", "kind", "width", "bb", "is_leader")}
        c = self._cols
        self.s = _Prog(prog["n_pcs"], prog["n_opcodes"], prog["n_bbs"], c["opcode"].ctypes.data,
                       c["kind"].ctypes.data, c["width"].ctypes.data, c["bb"].ctypes.data,
                       c["is_leader"].ctypes.data)

    def out(self, n_warps=0):
        p = self.prog
        return np.zeros(lib().orc_result_words(p["n_pcs"], p["n_opcodes"], p["n_bbs"], n_warps), dtype=np.int64)

    def unpack(self, out, n_warps=0):
        """Flat result words -> the numpy oracle's result dict."""
        p = self.prog
        P, O, B = p["n_pcs"], p["n_opcodes"], p["n_bbs"]
        r, k = {}, 0
        for name, n in (("counts", 4), ("H_t", O), ("H_w", O), ("Ent_t", B), ("Ent_w", B), ("Ins_t", B),
                        ("Ins_w", B), ("mem_n", P), ("mem_S", P), ("mem_L", P), ("hS", 33), ("hL", 33),
                        ("trace", 3)):
            r[name] = out[k:k + n].copy()
            k += n
        r["trace"] = r["trace"].view(np.uint64)
        if n_warps:
            r["PW_T"] = out[k:k + n_warps].copy()
            r["PW_W"] = out[k + n_warps:k + 2 * n_warps].copy()
        return r


def _check(rc, what):
    if rc != 0:
        raise RuntimeError(f"C oracle {what} failed (rc {rc})")


def _warps(w, total):
    return (0, total) if w is None else w


def events(prog, launch, warp, pc, A, P, addr=None, n_warps=0, trace=False):
    """EM §2 applied to an arbitrary event list (same as oracle.events.Accumulator.add)."""
    pr = Prog(prog)
    n = len(warp)
    cols = [np.ascontiguousarray(np.broadcast_to(np.asarray(x), (n,)), dtype=np.uint32) for x in (warp, pc, A, P)]
    ad = None if addr is None else np.ascontiguousarray(addr, dtype=np.uint64).reshape(n, 32)
    out = pr.out(n_warps)
    _check(lib().orc_events(C.byref(pr.s), launch, n, *(c.ctypes.data for c in cols),
                            None if ad is None else ad.ctypes.data, n_warps, int(trace), out.ctypes.data), "events")
    return pr.unpack(out, n_warps)


def sectors_lines(addr, E):
    a = np.ascontiguousarray(addr, dtype=np.uint64)
    S, L = C.c_uint32(), C.c_uint32()
    lib().orc_sectors_lines(a.ctypes.data, int(E), C.byref(S), C.byref(L))
    return S.value, L.value


def vectoradd(prog, N, a, b, c, launch=0, warps=None, threads=None, per_warp=False, trace=False):
    pr = Prog(prog)
    nw = -(-N // 256) * 8
    w0, w1 = _warps(warps, nw)
    npw = nw if per_warp else 0
    out = pr.out(npw)
    _check(lib().orc_vectoradd(C.byref(pr.s), N, a, b, c, launch, w0, w1, threads or host_threads(), npw,
                               int(trace), out.ctypes.data), "vectoradd")
    return pr.unpack(out, npw)


def sgemm(prog, M, N, K, A, B, Cp, launch=0, warps=None, threads=None, per_warp=False, trace=False):
    pr = Prog(prog)
    nw = -(-M // 32) * -(-N // 8) * 8
    w0, w1 = _warps(warps, nw)
    npw = nw if per_warp else 0
    out = pr.out(npw)
    _check(lib().orc_sgemm(C.byref(pr.s), M, N, K, A, B, Cp, launch, w0, w1, threads or host_threads(), npw,
                           int(trace), out.ctypes.data), "sgemm")
    return pr.unpack(out, npw)


def stencil(prog, n, buf0, buf1, iters, first_launch=0, warps=None, threads=None, trace=False):
    pr = Prog(prog)
    nw = -(-n // 32) * -(-n // 8) * 8
    w0, w1 = _warps(warps, nw)
    out = pr.out()
    _check(lib().orc_stencil(C.byref(pr.s), n, buf0, buf1, iters, first_launch, w0, w1, threads or host_threads(),
                             int(trace), out.ctypes.data), "stencil")
    return pr.unpack(out)


def bfs(prog, rowptr, col, src, ptrs, first_launch=0, warps=None, threads=None, per_warp=False, trace=False):
    """Whole BFS (EM §3.3). ptrs = (mask, visited, updating, cost, over, rowptr, col) device addresses.
    Returns (result dict, cost int32[n], levels)."""
    pr = Prog(prog)
    rp = np.ascontiguousarray(rowptr, dtype=np.int32)
    cl = np.ascontiguousarray(col, dtype=np.int32)
    n = len(rp) - 1
    nw = -(-n // 256) * 8
    w0, w1 = _warps(warps, nw)
    npw = nw if per_warp else 0
    out = pr.out(npw)
    pt = np.array(ptrs, dtype=np.uint64)
    cost = np.zeros(n, dtype=np.int32)
    levels = C.c_int64()
    _check(lib().orc_bfs(C.byref(pr.s), n, rp.ctypes.data, cl.ctypes.data, int(src), pt.ctypes.data, first_launch,
                         w0, w1, threads or host_threads(), npw, int(trace), out.ctypes.data, cost.ctypes.data,
                         C.byref(levels)), "bfs")
    return pr.unpack(out, npw), cost, levels.value


def gen_events(prog, seed, first, n):
    """Replay stream bytes of events [first, first + n): (headers u32[n, 4], addresses u64[n, 32])."""
    pr = Prog(prog)
    hdr = np.zeros((n, 4), dtype=np.uint32)
    addr = np.zeros((n, 32), dtype=np.uint64)
    lib().orc_gen_events(C.byref(pr.s), seed, first, n, hdr.ctypes.data, addr.ctypes.data)
    return hdr, addr


def replay(prog, seed, first, n, threads=None):
    """EM §3.5: events [first, first + n) of the generator, §2 items 1-4 applied to each."""
    pr = Prog(prog)
    out = pr.out()
    _check(lib().orc_replay(C.byref(pr.s), seed, first, n, threads or host_threads(), out.ctypes.data), "replay")
    return pr.unpack(out)
