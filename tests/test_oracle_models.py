"""Pins for oracle/programs.py, oracle/models/*, oracle/gen.py, oracle/trace.py.

Closed forms here are derived by hand from docs/EVENT_MODEL.md §3 (derivations in comments) and are
independent of the oracle's code paths."""
import json
import os

import numpy as np
import pytest

from oracle import events as ev, programs, gen, trace
from oracle.models import vectoradd, sgemm, stencil, bfs
from synth import rmat_csr, bfs_source

GOLD = os.path.join(os.path.dirname(__file__), "golden")
OPN = ["S2R", "IMAD", "ISETP", "EXIT", "IMAD.WIDE", "LDG", "STG", "FADD", "FFMA", "MOV", "IADD", "BRA", "SEL"]
BASE = 1 << 32  # 128-byte aligned buffer bases


# ---------------------------------------------------------------- programs: BB rule (R-14)
@pytest.mark.parametrize("name", ["vectoradd", "sgemm", "bfs", "stencil", "replay", "wfft_emu", "wfft_sw"])
def test_bb_rule(name):
    p = getattr(programs, name)()
    n = p["n_pcs"]
    targets = {int(t) for t in p["target"] if t >= 0}
    for pc in range(n):
        starts = pc == 0 or p["kind"][pc - 1] == programs.CTRL or pc in targets or p["bb"][pc] != p["bb"][pc - 1]
        if name == "replay":
            assert p["is_leader"][pc] == (pc % 8 == 0)
            continue
        # a new block starts exactly after a control-flow instruction or at a branch target
        expect_new = pc == 0 or p["kind"][pc - 1] == programs.CTRL or pc in targets
        assert bool(p["is_leader"][pc]) == expect_new, (name, pc)
        assert (pc == 0 or p["bb"][pc] != p["bb"][pc - 1]) == expect_new, (name, pc)
    assert p["bb"].max() + 1 == p["n_bbs"]


# ---------------------------------------------------------------- C1 closed forms (I-3, C-15)
@pytest.mark.parametrize("N", [65536, 65500])
def test_vectoradd_closed_form(N):
    g = json.load(open(os.path.join(GOLD, "vectoradd_closed_form.json")))["N%d" % N]
    prog = programs.vectoradd()
    acc = ev.Accumulator(prog, n_warps=vectoradd.n_warps(N))
    vectoradd.run(acc, N, BASE, BASE + (1 << 20), BASE + (2 << 20))
    r = acc.result()
    assert r["counts"].tolist() == [g["T_issued"], g["T_exec"], g["W_issued"], g["W_exec"]]
    if "H_t" in g:
        for name, v in g["H_t"].items():
            assert r["H_t"][OPN.index(name)] == v, name
        for pc in (7, 8, 11):
            m = g["mem_per_pc"]
            assert r["mem_n"][pc] == m["n"]
            assert r["mem_S"][pc] == m["n"] * m["S_per_event"]
            assert r["mem_L"][pc] == m["n"] * m["L_per_event"]
    else:
        # warp 2046: 28 live lanes after pc4 (A = 0x0FFFFFFF), 112 contiguous bytes -> S = 4, L = 1
        acc2 = ev.Accumulator(prog)
        vectoradd.run(acc2, N, BASE, BASE, BASE, warps=[2046])
        r2 = acc2.result()
        assert r2["mem_S"][7] == g["warp2046_S"] and r2["mem_L"][7] == g["warp2046_L"]
        assert r2["counts"][0] == 5 * 32 + 8 * bin(int(g["warp2046_A_after_exit"], 16)).count("1")
    assert ev.invariants(r) == []
    # BB: BB0 entered by every warp with all lanes, BB1 by warps with live lanes
    assert r["Ent_w"][0] == vectoradd.n_warps(N)


# ---------------------------------------------------------------- C2 closed forms (I-3)
@pytest.mark.parametrize("M,N,K", [(64, 32, 48), (32, 64, 33)])
def test_sgemm_closed_form(M, N, K):
    # M%32 == N%8 == 0, K >= 32, N >= 32: A and C accesses are 32 distinct lines, B is a broadcast.
    W = M * N // 32
    acc = ev.Accumulator(programs.sgemm(), n_warps=W)
    sgemm.run(acc, M, N, K, BASE, BASE + (1 << 24), BASE + (2 << 24))
    r = acc.result()
    w_iss = W * (10 + 6 * K + 2)
    w_exe = w_iss - W - W                      # @P0 EXIT never executes; last @P1 BRA predicated off
    assert r["counts"].tolist() == [32 * w_iss, 32 * w_exe, w_iss, w_exe]
    assert r["mem_n"][10] == W * K and r["mem_S"][10] == W * K * 32 and r["mem_L"][10] == W * K * 32
    assert r["mem_n"][11] == W * K and r["mem_S"][11] == W * K and r["mem_L"][11] == W * K
    assert r["mem_n"][16] == W and r["mem_S"][16] == 32 * W and r["mem_L"][16] == 32 * W
    assert r["Ent_w"][2] == W * K and r["Ins_w"][2] == W * (6 * K - 1)
    assert r["hS"][32] == W * (K + 1) and r["hS"][1] == W * K
    assert ev.invariants(r) == []


def test_sgemm_full_size_formula_matches_survey():
    # SURVEY I-3: 67,141,632 mem events, sum S = sum L = 1,108,344,832 at M = N = K = 1024
    W, K = 1024 * 1024 // 32, 1024
    assert W * (2 * K + 1) == 67_141_632
    assert W * K * 32 + W * K + 32 * W == 1_108_344_832


def test_sgemm_ragged_invariants():
    M, N, K = 100, 20, 5
    acc = ev.Accumulator(programs.sgemm(), n_warps=sgemm.n_warps(M, N))
    sgemm.run(acc, M, N, K, BASE, BASE + (1 << 24), BASE + (2 << 24))
    r = acc.result()
    assert ev.invariants(r) == []
    assert r["PW_T"].sum() == r["counts"][1]
    # live lanes: M*N threads execute 6K-1+... ; the exec count of the A-load is exactly M*N*K
    assert r["H_t"][OPN.index("LDG")] == 2 * M * N * K
    assert r["H_t"][OPN.index("STG")] == M * N


# ---------------------------------------------------------------- C4 closed forms (I-3)
def stencil_closed_form(n):
    G = n // 32
    W = n * n // 32
    rec = 2 * W + 4 * (n - 2) * G
    S = 8 * G * n + (n - 2) * (18 * G - 2)
    L = 2 * G * n + (n - 2) * (6 * G - 2)
    t_exec = 12 * n * n + 8 * (n - 2) ** 2
    w_iss = 21 * W
    w_exe = w_iss - W - 8 * 2 * G
    return rec, S, L, t_exec, w_iss, w_exe


@pytest.mark.parametrize("n", [64, 96])
def test_stencil_closed_form(n):
    acc = ev.Accumulator(programs.stencil(), trace=True)
    stencil.run_iterations(acc, n, BASE, BASE + (1 << 24), iters=2)
    r = acc.result()
    rec, S, L, t_exec, w_iss, w_exe = stencil_closed_form(n)
    assert int(r["trace"][0]) == 2 * rec == r["mem_n"].sum()
    assert r["mem_S"].sum() == 2 * S and r["mem_L"].sum() == 2 * L
    assert r["counts"].tolist() == [2 * 32 * w_iss, 2 * t_exec, 2 * w_iss, 2 * w_exe]
    assert ev.invariants(r) == []


def test_stencil_full_size_formula_matches_survey():
    rec, S, L, *_ = stencil_closed_form(8192)
    assert (rec, S, L) == (12_580_864, 54_500_356, 16_757_764)   # SURVEY I-3 per iteration


# ---------------------------------------------------------------- C3 BFS (I-4 + hand-checked launch)
def test_bfs_distances_match_scipy():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import shortest_path
    rowptr, col = rmat_csr(10, 8, seed=5)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    acc = ev.Accumulator(programs.bfs())
    ptr = bfs.Ptrs(*(BASE + (k << 24) for k in range(7)))
    cost, levels, launches = bfs.run(acc, rowptr, col, src, ptr)
    G = csr_matrix((np.ones(len(col)), col, rowptr), shape=(n, n))
    d = shortest_path(G, unweighted=True, indices=src)
    exp = np.where(np.isinf(d), -1, d).astype(np.int64)
    assert (cost.astype(np.int64) == exp).all()
    assert launches == 2 * levels
    r = acc.result()
    assert ev.invariants(r) == []
    # K1 writes updating[nb] once per (frontier vertex, unvisited neighbour) pair, K2 once per new vertex
    assert r["H_w"].sum() == r["counts"][3]


def test_bfs_path_graph_hand_checked():
    # n = 3, edges 0-1 and 1-2, source 1 (max degree). Level 0, kernel 1, one warp:
    # pcs 0-4 (5 events, pc4 executed by lanes 3..31), pcs 5-7 (A = 0b111, pc7 executed by lanes 0, 2),
    # pcs 8-12 (A = 0b010, pc12 predicated off), loop k = 0, 1 (8 events each; pc16 off both times,
    # pc20 executed at k = 0 only), pc21. -> 30 warp events, 26 executed.
    rowptr = np.array([0, 1, 3, 4], dtype=np.int32)
    col = np.array([1, 0, 2, 1], dtype=np.int32)
    acc = ev.Accumulator(programs.bfs())
    ptr = bfs.Ptrs(*(BASE + (k << 24) for k in range(7)))
    st = {"mask": np.array([0, 1, 0], np.uint8), "visited": np.array([0, 1, 0], np.uint8),
          "updating": np.zeros(3, np.uint8)}
    bfs.kernel1(acc, 0, np.array([0]), rowptr.astype(np.int64), col.astype(np.int64), st, ptr)
    r = acc.result()
    assert r["counts"][2] == 30 and r["counts"][3] == 26
    t_iss = 5 * 32 + 3 * 3 + 5 * 1 + 16 * 1 + 3
    t_exe = 4 * 32 + 29 + 2 * 3 + 2 + 4 * 1 + (8 - 1) * 1 + (8 - 2) * 1 + 3
    assert r["counts"][0] == t_iss and r["counts"][1] == t_exe
    assert r["mem_n"][17] == 2                 # both neighbours unvisited -> updating[0], updating[2]


# ---------------------------------------------------------------- C5 generator
def test_generator_properties():
    prog = programs.replay()
    pc, warp, A, P, addr = gen.events(0, 20000, prog)
    assert (A != 0).all() and (pc < 4096).all() and (warp < (1 << 20)).all()
    mem = programs.is_mem(prog)[pc]
    wd = prog["width"][pc[mem]].astype(np.uint64)[:, None]
    assert ((addr[mem] % wd) == 0).all()                       # aligned (R-7)
    assert (addr[~mem] == 0).all()
    assert 0.2 < programs.is_mem(prog).mean() < 0.3
    S, L = ev.sectors_lines(addr[mem], A[mem] & P[mem])
    E0 = (A[mem] & P[mem]) == 0
    assert S[~E0].min() == 1 and S.max() == 32                 # S spans 1..32
    # (E = 0 needs two random masks to be disjoint, p ~ 1e-5 per event: C-10 is exercised by C1-C4)
    # partition invariance: any sub-range regenerates identical events
    pc2, warp2, A2, P2, addr2 = gen.events(12345, 500, prog)
    assert (pc2 == pc[12345:12845]).all() and (addr2 == addr[12345:12845]).all()
    assert (A2 == A[12345:12845]).all() and (P2 == P[12345:12845]).all()


def test_replay_partition_additivity():
    prog = programs.replay()
    a, b = ev.Accumulator(prog), ev.Accumulator(prog)
    gen.replay(a, 0, 6000)
    gen.replay(b, 0, 2500)
    gen.replay(b, 2500, 3500)
    ra, rb = a.result(), b.result()
    for k in ra:
        assert (ra[k] == rb[k]).all(), k
    assert ev.invariants(ra) == []


# ---------------------------------------------------------------- trace records and digests
def test_record_layout_by_hand():
    prog = programs.vectoradd()
    addr = np.arange(32, dtype=np.uint64)[None, :] * 4 + np.uint64(0x1000)
    rec = trace.build_records(7, np.array([9]), np.array([2]), np.array([11]), np.array([0xF0F0F0F0]),
                              np.array([0xFFFF0000]), prog, addr, np.array([0xF0F00000]))
    b = rec[0].tobytes()
    u32 = lambda o: int.from_bytes(b[o:o + 4], "little")
    assert (u32(0), u32(4), u32(8), u32(12), u32(16), u32(20)) == (7, 9, 2, 11, 0xF0F0F0F0, 0xFFFF0000)
    assert int.from_bytes(b[24:26], "little") == 6 and b[26] == 4 and b[27] == programs.GST
    assert u32(28) == 0
    for l in range(32):
        a = int.from_bytes(b[32 + 8 * l:40 + 8 * l], "little")
        assert a == ((0x1000 + 4 * l) if (0xF0F00000 >> l) & 1 else 0)


def test_digest_order_independent_and_sensitive():
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    stencil.run(acc, 64, BASE, BASE + (1 << 24))
    recs = acc.record_array()
    d = trace.Digest(); d.update(recs)
    rng = np.random.default_rng(0)
    d2 = trace.Digest(); d2.update(recs[rng.permutation(len(recs))])
    assert (d.n, d.d1, d.d2) == (d2.n, d2.d1, d2.d2) == (acc.digest.n, acc.digest.d1, acc.digest.d2)
    for byte in (0, 13, 27, 100, 287):
        r2 = recs.copy(); r2[5, byte] ^= 1
        d3 = trace.Digest(); d3.update(r2)
        assert d3.d1 != d.d1 and d3.d2 != d.d2
    # seq numbers are 0.. per (launch, warp)
    r = recs.view(trace.RECORD_DTYPE).reshape(-1)
    w0 = r[r["warp"] == 300]
    assert sorted(w0["seq"].tolist()) == list(range(len(w0)))


def test_footprint_brute_force():
    """F2 footprint vs Python sets over random records (two launches, random masks, clustered addresses)."""
    rng = np.random.default_rng(11)
    n = 300
    rec = np.zeros(n, dtype=trace.RECORD_DTYPE)
    rec["launch"] = rng.integers(0, 3, n)
    rec["A"] = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    rec["P"] = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    rec["addr"] = (0x7f0000000000 + rng.integers(0, 1 << 14, (n, 32))).astype(np.uint64)
    got = trace.footprint(rec.view(np.uint8).reshape(n, -1), 4)
    for l in range(4):
        secs, lines, cnt = set(), set(), 0
        for r in rec:
            if int(r["launch"]) != l:
                continue
            cnt += 1
            e = int(r["A"]) & int(r["P"])
            for lane in range(32):
                if (e >> lane) & 1:
                    secs.add(int(r["addr"][lane]) // 32)
                    lines.add(int(r["addr"][lane]) // 128)
        assert list(got[l]) == [len(secs), len(lines), cnt]


@pytest.mark.parametrize("N", [1, 31, 1000, 4097])
def test_footprint_vectoradd_closed_form(N):
    """vectorAdd touches three disjoint 128 B-aligned arrays of 4N bytes: 3*ceil(4N/32) sectors and
    3*ceil(4N/128) lines in its single launch."""
    acc = ev.Accumulator(programs.vectoradd(), trace=True, keep_records=True)
    vectoradd.run(acc, N, 0x100000, 0x200000, 0x300000)
    fp = trace.footprint(acc.record_array(), 1)
    assert list(fp[0][:2]) == [3 * -(-4 * N // 32), 3 * -(-4 * N // 128)]
