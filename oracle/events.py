"""Per-event definitions — docs/EVENT_MODEL.md §2, applied event by event.

`Accumulator.add(...)` receives a batch of events that share nothing but the call (a batch is just a
list of independent events; every sum below is a sum of non-negative integers, so batching cannot
change a result). Nothing here is blocked, fused or reordered beyond that.
"""
from __future__ import annotations

import numpy as np

from .programs import MEM_KINDS
from . import trace as _trace

SENTINEL = np.uint64((1 << 64) - 1)  # never equal to addr >> 5 or addr >> 7


def popc(x):
    """Population count of uint32 masks."""
    return np.bitwise_count(np.asarray(x, dtype=np.uint32)).astype(np.int64)


def lane_bits(mask):
    """[n] uint32 masks -> [n, 32] bool, column l = bit l."""
    m = np.asarray(mask, dtype=np.uint64)[:, None]
    return ((m >> np.arange(32, dtype=np.uint64)[None, :]) & np.uint64(1)).astype(bool)


def distinct_count(keys, active):
    """|{keys[r, l] : active[r, l]}| for every row r (keys uint64 [n, 32], active bool [n, 32])."""
    k = np.where(active, keys, SENTINEL)
    k = np.sort(k, axis=1)
    new = np.ones(k.shape, dtype=bool)
    new[:, 1:] = k[:, 1:] != k[:, :-1]
    return (new & (k != SENTINEL)).sum(axis=1).astype(np.int64)


def sectors_lines(addr, E):
    """§2 item 4: S = distinct addr>>5 over lanes of E, L = distinct addr>>7 (readings R-3, R-6)."""
    act = lane_bits(E)
    a = np.asarray(addr, dtype=np.uint64)
    return distinct_count(a >> np.uint64(5), act), distinct_count(a >> np.uint64(7), act)


class Accumulator:
    """Cumulative results for one program (EVENT_MODEL §4)."""

    def __init__(self, prog, n_warps=None, trace=False, keep_records=False):
        self.prog = prog
        P, O, B = prog["n_pcs"], prog["n_opcodes"], prog["n_bbs"]
        self.counts = np.zeros(4, dtype=np.int64)            # T_issued, T_exec, W_issued, W_exec
        self.H_t = np.zeros(O, dtype=np.int64)
        self.H_w = np.zeros(O, dtype=np.int64)
        self.Ent_t = np.zeros(B, dtype=np.int64)
        self.Ent_w = np.zeros(B, dtype=np.int64)
        self.Ins_t = np.zeros(B, dtype=np.int64)
        self.Ins_w = np.zeros(B, dtype=np.int64)
        self.mem_n = np.zeros(P, dtype=np.int64)
        self.mem_S = np.zeros(P, dtype=np.int64)
        self.mem_L = np.zeros(P, dtype=np.int64)
        self.hS = np.zeros(33, dtype=np.int64)
        self.hL = np.zeros(33, dtype=np.int64)
        self.n_warps = n_warps
        if n_warps is not None:
            self.PW_T = np.zeros(n_warps, dtype=np.int64)
            self.PW_W = np.zeros(n_warps, dtype=np.int64)
        self.trace = trace
        self.digest = _trace.Digest()
        self.records = [] if keep_records else None
        self._seq = {}

    # ------------------------------------------------------------------ events
    def add(self, launch, warp, pc, A, P, addr=None):
        """Apply §2 to a batch of events.

        launch: int; warp, A, P: arrays [n]; pc: int or array [n];
        addr: uint64 [n, 32] or None (required when pc is a global-memory pc).
        Events with A == 0 are not events (§1) and are dropped here.
        """
        warp = np.asarray(warp, dtype=np.int64)
        A = np.asarray(A, dtype=np.uint64).astype(np.uint32)
        n = len(warp)
        pc = np.broadcast_to(np.asarray(pc, dtype=np.int64), (n,))
        keep = A != 0
        if not keep.all():
            warp, A, pc = warp[keep], A[keep], pc[keep]
            P = np.asarray(P)[keep]
            if addr is not None:
                addr = np.asarray(addr)[keep]
        if len(warp) == 0:
            return
        P = np.asarray(P, dtype=np.uint64).astype(np.uint32)
        E = A & P                                   # reading R-1: E = A & P
        pA, pE = popc(A), popc(E)
        ex = (E != 0).astype(np.int64)
        prog = self.prog
        # 1. counts (Listing 1; R-9)
        self.counts[0] += pA.sum()
        self.counts[1] += pE.sum()
        self.counts[2] += len(warp)
        self.counts[3] += ex.sum()
        if self.n_warps is not None:
            np.add.at(self.PW_T, warp, pE)
            np.add.at(self.PW_W, warp, ex)
        # 2. opcode histogram (§6.2)
        op = prog["opcode"][pc]
        np.add.at(self.H_t, op, pE)
        np.add.at(self.H_w, op, ex)
        # 3. basic blocks
        b = prog["bb"][pc]
        np.add.at(self.Ins_t, b, pE)
        np.add.at(self.Ins_w, b, ex)
        lead = prog["is_leader"][pc] == 1
        np.add.at(self.Ent_t, b[lead], pA[lead])
        np.add.at(self.Ent_w, b[lead], 1)
        # 4. memory divergence (Listing 8)
        mem = np.isin(prog["kind"][pc], MEM_KINDS) & (E != 0)
        if mem.any():
            if addr is None:
                raise ValueError("memory events need addresses")
            addr = np.asarray(addr, dtype=np.uint64)
            mpc, mE, ma = pc[mem], E[mem], addr[mem]
            S, L = sectors_lines(ma, mE)
            np.add.at(self.mem_n, mpc, 1)
            np.add.at(self.mem_S, mpc, S)
            np.add.at(self.mem_L, mpc, L)
            np.add.at(self.hS, S, 1)
            np.add.at(self.hL, L, 1)
            # 5. trace records (§5)
            if self.trace:
                mw, mA, mP = warp[mem], A[mem], P[mem]
                seq = np.empty(len(mw), dtype=np.int64)
                for r, w in enumerate(mw.tolist()):
                    key = (launch, w)
                    seq[r] = self._seq.get(key, 0)
                    self._seq[key] = seq[r] + 1
                recs = _trace.build_records(launch, mw, seq, mpc, mA, mP, prog, ma, mE)
                self.digest.update(recs)
                if self.records is not None:
                    self.records.append(recs)

    # ------------------------------------------------------------------ results
    def record_array(self):
        if not self.records:
            return np.zeros((0, _trace.RECORD_BYTES), dtype=np.uint8)
        return np.concatenate(self.records)

    def result(self):
        r = {
            "counts": self.counts.copy(),
            "H_t": self.H_t.copy(), "H_w": self.H_w.copy(),
            "Ent_t": self.Ent_t.copy(), "Ent_w": self.Ent_w.copy(),
            "Ins_t": self.Ins_t.copy(), "Ins_w": self.Ins_w.copy(),
            "mem_n": self.mem_n.copy(), "mem_S": self.mem_S.copy(), "mem_L": self.mem_L.copy(),
            "hS": self.hS.copy(), "hL": self.hL.copy(),
            "trace": np.array([self.digest.n, self.digest.d1, self.digest.d2], dtype=np.uint64),
        }
        if self.n_warps is not None:
            r["PW_T"] = self.PW_T.copy()
            r["PW_W"] = self.PW_W.copy()
        return r


def invariants(r):
    """I-2 — returns a list of violated invariant names (empty = all hold)."""
    bad = []
    Ti, Te, Wi, We = (int(x) for x in r["counts"])
    if not We <= Wi: bad.append("W_exec<=W_issued")
    if not (We <= Te <= 32 * We): bad.append("W_exec<=T_exec<=32W_exec")
    if not (Te <= Ti <= 32 * Wi): bad.append("T_exec<=T_issued<=32W_issued")
    if r["H_t"].sum() != Te or r["H_w"].sum() != We: bad.append("sum H = totals")
    if r["Ins_t"].sum() != Te or r["Ins_w"].sum() != We: bad.append("sum Ins = totals")
    if r["hS"].sum() != r["mem_n"].sum() or r["hL"].sum() != r["mem_n"].sum(): bad.append("sum hist = n")
    if r["hS"][0] != 0 or r["hL"][0] != 0: bad.append("S,L >= 1")
    if not (r["mem_L"] <= r["mem_S"]).all() or not (r["mem_S"] <= 4 * r["mem_L"]).all(): bad.append("L<=S<=4L")
    if not (r["mem_n"] <= r["mem_L"]).all() or not (r["mem_S"] <= 32 * r["mem_n"]).all(): bad.append("1<=S<=32")
    return bad
