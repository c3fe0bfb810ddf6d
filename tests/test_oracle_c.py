"""Pins for the multithreaded C oracle (oracle/c/nvbt_oracle.c via oracle/coracle.py) — CPU only.

The C oracle is the second, independent transcription of docs/EVENT_MODEL.md that makes full-size
parity affordable. It is pinned here against things other than itself:
  * the numpy oracle (pinned in tests/test_oracle_*.py by brute force, the paper's Listing 8 example,
    published splitmix64 outputs and closed forms), element by element, on every workload at several
    sizes (ragged tails, trace digests, per-warp arrays) and on random event lists;
  * Python set definitions of S and L (EM §2 item 4; P:L263 (§6.1)) on random and adversarial lanes;
  * SURVEY §8(c) I-3 closed forms at BASELINE.json's full sizes (SGEMM 1024^3; one 8192^2 stencil
    iteration) and a closed form of the stencil derived for any n (comment below);
  * thread-count invariance (the split over host threads must not change a result, EM §4).
"""
import numpy as np
import pytest

from oracle import coracle as co, events as ev, programs, gen
from oracle.models import vectoradd as m_va, sgemm as m_sg, stencil as m_st, bfs as m_bfs
from synth import rmat_csr, bfs_source

BASE = 1 << 32


def same(c, o, what):
    for k in o:
        if k in c:
            a, b = np.asarray(c[k]).astype(np.int64), np.asarray(o[k]).astype(np.int64)
            assert a.shape == b.shape and np.array_equal(a, b), (what, k, a, b)


# ---------------------------------------------------------------- S / L against set definitions
def test_sectors_lines_sets():
    rng = np.random.default_rng(11)
    for trial in range(3000):
        scale = [4, 32, 128, 4096, 1 << 20, 1 << 40][trial % 6]
        base = int(rng.integers(0, 1 << 40))
        width = [1, 2, 4, 8, 16][trial % 5]
        addr = [((base + int(o)) // width) * width for o in rng.integers(0, scale, 32)]
        if trial % 7 == 0:
            addr = sorted(addr)
        E = int(rng.integers(0, 1 << 32)) if trial % 3 else 0xFFFFFFFF
        S, L = co.sectors_lines(addr, E)
        lanes = [l for l in range(32) if E >> l & 1]
        assert S == len({addr[l] >> 5 for l in lanes}) and L == len({addr[l] >> 7 for l in lanes}), (addr, E)


def test_sectors_lines_paper_example():
    """two threads on the same cache line each add 1/2 -> one line; here S = L = 1."""
    assert co.sectors_lines([BASE + 4, BASE + 8] + [0] * 30, 0b11) == (1, 1)
    assert co.sectors_lines([BASE, BASE + 32, BASE + 128] + [0] * 29, 0b111) == (3, 2)


# ---------------------------------------------------------------- random event lists vs numpy
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_events_match_numpy(seed):
    rng = np.random.default_rng(seed)
    for prog in (programs.replay(), programs.bfs(), programs.stencil()):
        n = 3000
        pc = rng.integers(0, prog["n_pcs"], n)
        warp = rng.integers(0, 40, n)
        A = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
        A[rng.random(n) < 0.3] = 0xFFFFFFFF
        A[rng.random(n) < 0.05] = 0                        # not events (EM §1)
        P = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
        P[rng.random(n) < 0.5] = 0xFFFFFFFF
        base = rng.integers(0, 1 << 40, n, dtype=np.uint64)[:, None]
        scale = np.array([4, 128, 4096, 1 << 30], dtype=np.uint64)[rng.integers(0, 4, n)][:, None]
        addr = (base + rng.integers(0, 1 << 62, (n, 32), dtype=np.uint64) % scale) & ~np.uint64(3)
        acc = ev.Accumulator(prog, n_warps=40, trace=True)
        acc.add(5, warp, pc, A, P, addr)
        c = co.events(prog, 5, warp, pc, A, P, addr, n_warps=40, trace=True)
        same(c, acc.result(), f"random events {seed}")


# ---------------------------------------------------------------- workloads vs numpy (small sizes)
@pytest.mark.parametrize("N", [65536, 65500, 1000, 31, 257])
def test_vectoradd_matches_numpy(N):
    p = programs.vectoradd()
    acc = ev.Accumulator(p, n_warps=m_va.n_warps(N), trace=True)
    m_va.run(acc, N, BASE, BASE + (1 << 20), BASE + (2 << 20) + 4, launch=3)
    same(co.vectoradd(p, N, BASE, BASE + (1 << 20), BASE + (2 << 20) + 4, launch=3, per_warp=True, trace=True),
         acc.result(), f"vectorAdd {N}")


@pytest.mark.parametrize("M,N,K", [(64, 32, 48), (100, 20, 5), (33, 9, 1), (96, 64, 130)])
def test_sgemm_matches_numpy(M, N, K):
    p = programs.sgemm()
    acc = ev.Accumulator(p, n_warps=m_sg.n_warps(M, N), trace=True)
    m_sg.run(acc, M, N, K, BASE, BASE + (1 << 24) + 64, BASE + (2 << 24))
    same(co.sgemm(p, M, N, K, BASE, BASE + (1 << 24) + 64, BASE + (2 << 24), per_warp=True, trace=True),
         acc.result(), f"SGEMM {M}x{N}x{K}")


@pytest.mark.parametrize("n,iters", [(96, 3), (100, 2), (64, 1), (33, 2)])
def test_stencil_matches_numpy(n, iters):
    p = programs.stencil()
    acc = ev.Accumulator(p, trace=True)
    m_st.run_iterations(acc, n, BASE, BASE + (1 << 26), iters, first_launch=2)
    same(co.stencil(p, n, BASE, BASE + (1 << 26), iters, first_launch=2, trace=True), acc.result(), f"stencil {n}")


@pytest.mark.parametrize("scale", [8, 10, 12])
def test_bfs_matches_numpy(scale):
    p = programs.bfs()
    rp, cl = rmat_csr(scale, 16, seed=3)
    src = bfs_source(rp)
    ptr = [BASE + k * (1 << 24) for k in range(7)]
    acc = ev.Accumulator(p, n_warps=m_bfs.n_warps(len(rp) - 1), trace=True)
    c1, l1, _ = m_bfs.run(acc, rp, cl, src, m_bfs.Ptrs(*ptr))
    r, c2, l2 = co.bfs(p, rp, cl, src, ptr, per_warp=True, trace=True)
    assert l1 == l2 and np.array_equal(c1, c2)
    same(r, acc.result(), f"BFS scale {scale}")


@pytest.mark.parametrize("first,n", [(0, 1 << 16), (123456789, 50_003), (10**10 - 20000, 20000)])
def test_replay_matches_numpy(first, n):
    p = programs.replay()
    acc = ev.Accumulator(p)
    gen.replay(acc, first, n)
    same(co.replay(p, gen.SEED, first, n), acc.result(), f"replay {first}+{n}")


def test_generator_bytes_match_numpy():
    p = programs.replay()
    for first, n in [(0, 4096), (10**10 - 4099, 4099)]:
        h, a = co.gen_events(p, gen.SEED, first, n)
        pc, w, A, P, ad = gen.events(first, n)
        assert (h[:, 0] == pc).all() and (h[:, 1] == w).all() and (h[:, 2] == A).all() and (h[:, 3] == P).all()
        assert (a == ad).all()


def test_thread_count_invariance():
    p = programs.replay()
    r = [co.replay(p, gen.SEED, 777, 200_001, threads=t) for t in (1, 3, 8)]
    same(r[1], r[0], "replay 3 threads")
    same(r[2], r[0], "replay 8 threads")
    s = programs.stencil()
    a = co.stencil(s, 200, BASE, BASE + (1 << 24), 2, trace=True, threads=1)
    b = co.stencil(s, 200, BASE, BASE + (1 << 24), 2, trace=True, threads=7)
    same(b, a, "stencil 7 threads")


# ---------------------------------------------------------------- closed forms at full size (I-3)
def test_sgemm_full_size_closed_form():
    """SURVEY I-3 at 1024^3 (EM §3.2 program): 32,768 warps; mem events 32,768 x (2K + 1) = 67,141,632;
    A loads 32 sectors / 32 lines (4096 B lane stride), B loads 1 / 1 (broadcast), C stores 32 / 32, so
    ΣS = ΣL = 32,768 x (1024 x 33 + 32) = 1,108,344,832; every warp issues 12 + 6K warp instructions and
    executes all but the never-taken `@P0 EXIT` and the last `@P1 BRA`."""
    M = N = K = 1024
    r = co.sgemm(programs.sgemm(), M, N, K, BASE, BASE + (4 << 20), BASE + (8 << 20))
    W = 32768
    assert int(r["mem_n"].sum()) == 67_141_632
    assert int(r["mem_S"].sum()) == int(r["mem_L"].sum()) == 1_108_344_832
    w_iss = W * (12 + 6 * K)
    assert r["counts"].tolist() == [32 * w_iss, 32 * (w_iss - 2 * W), w_iss, w_iss - 2 * W]


def stencil_closed_form(n, iters):
    """EM §3.4 with 128 B-aligned rows (n % 32 == 0), G = n/32 warps per row. Rows 0 and n-1: P1 = 0, so
    only the center load and the store execute: 2 records, (S, L) = (4, 1) each. Interior rows: 6 records;
    center/up/down/store (4, 1) each, left/right (5, 2) for interior warps; the first warp of a row loses
    lane j = 0 (left touches only its own line: 4/1) and the last loses j = n-1 (right 4/1), so edge
    warps total 25/7 and interior warps 26/8 (SURVEY I-3)."""
    G = n // 32
    rec = 4 * G + 6 * G * (n - 2)
    S = 16 * G + (n - 2) * (2 * 25 + (G - 2) * 26)
    L = 4 * G + (n - 2) * (2 * 7 + (G - 2) * 8)
    return iters * rec, iters * S, iters * L


def test_stencil_closed_form_formula_matches_survey():
    assert stencil_closed_form(8192, 1) == (12_580_864, 54_500_356, 16_757_764)
    assert stencil_closed_form(8192, 100) == (1_258_086_400, 5_450_035_600, 1_675_776_400)


@pytest.mark.parametrize("n,iters", [(1024, 3), (8192, 1)])
def test_stencil_closed_form(n, iters):
    r = co.stencil(programs.stencil(), n, BASE, BASE + (1 << 30), iters, trace=True)
    rec, S, L = stencil_closed_form(n, iters)
    assert int(r["trace"][0]) == rec and int(r["mem_n"].sum()) == rec
    assert int(r["mem_S"].sum()) == S and int(r["mem_L"].sum()) == L


def test_ent_t_guarded_leader_golden():
    """tests/golden/guarded_leader.json through the C oracle (Ent_t counts A, not E, at a guarded leader)."""
    from tests.test_oracle_events import guarded_leader_case
    prog, c, exp = guarded_leader_case()
    r = co.events(prog, 0, np.zeros(len(c["pc"]), dtype=np.uint32), c["pc"], c["A"], c["P"], c["addr"])
    for k in ("Ent_t", "Ent_w", "Ins_t", "Ins_w", "counts"):
        assert r[k].tolist() == exp[k], k
