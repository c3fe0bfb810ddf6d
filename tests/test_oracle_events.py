"""Pins for oracle/events.py and oracle/mix.py. CPU only."""
import itertools
import json
import os
from fractions import Fraction

import numpy as np
import pytest

from oracle import events as ev
from oracle.mix import mix64, mix64_int, R, K

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ALPHABET = [0, 4, 32, 36, 96, 128, 160, 4096]


def tiny_prog():
    # pc0: ALU (leader of bb0), pc1: GLD width 4 (bb0), pc2: GST (leader of bb1)
    return {
        "opcode": np.array([3, 5, 6]), "kind": np.array([0, 2, 3]), "width": np.array([0, 4, 4]),
        "bb": np.array([0, 0, 1]), "is_leader": np.array([1, 0, 1]), "guarded": np.array([1, 1, 1]),
        "n_pcs": 3, "n_opcodes": 8, "n_bbs": 2,
    }


def bits(x, w):
    return [l for l in range(w) if (x >> l) & 1]


# ---------------------------------------------------------------- mix64 pins
def test_mix64_published_vectors():
    g = json.load(open(os.path.join(GOLD, "splitmix64.json")))
    assert mix64_int(0) == int(g["state0_first"], 16)
    s, out = 1234567, []
    for _ in range(5):
        out.append(mix64_int(s))
        s = (s + 0x9E3779B97F4A7C15) % (1 << 64)
    assert out == g["seed1234567_first5"]


def test_mix64_numpy_matches_int():
    xs = [0, 1, 2**63, 2**64 - 1, 0x9E3779B97F4A7C15, 123456789012345678]
    got = mix64(np.array(xs, dtype=np.uint64))
    assert [int(v) for v in got] == [mix64_int(x) for x in xs]
    assert int(R(np.uint64(5), 3)) == mix64_int(K(3) ^ 5)


# ---------------------------------------------------------------- I-1 brute force
def brute_event(A, P, addr, w):
    """Plain-Python §2 for one event on a w-lane warp."""
    E = A & P
    lanes = bits(E, w)
    S = len({addr[l] >> 5 for l in lanes})
    L = len({addr[l] >> 7 for l in lanes})
    return bin(A).count("1"), bin(E).count("1"), int(E != 0), S, L


@pytest.mark.parametrize("w", [1, 2, 3, 4, 5])
def test_brute_force_all_masks(w):
    rng = np.random.default_rng(w)
    prog = tiny_prog()
    cases = []
    for A in range(1, 1 << w):
        for P in range(0, 1 << w):           # includes P bits outside A (must be masked away)
            if w <= 3:
                for combo in itertools.product(ALPHABET, repeat=w):
                    cases.append((A, P, list(combo)))
            else:
                for _ in range(6):
                    cases.append((A, P, list(rng.choice(ALPHABET, size=w))))
    acc = ev.Accumulator(prog, n_warps=1)
    exp = np.zeros(4, dtype=np.int64)
    eS = np.zeros(3, dtype=np.int64)
    eL = np.zeros(3, dtype=np.int64)
    en = np.zeros(3, dtype=np.int64)
    hS = np.zeros(33, dtype=np.int64)
    for A, P, a in cases:
        addr = np.zeros((1, 32), dtype=np.uint64)
        addr[0, :w] = a
        for pc in (0, 1, 2):
            acc.add(0, [0], pc, [A], [P], addr if pc else None)
            pA, pE, ex, S, L = brute_event(A, P, a, w)
            exp += [pA, pE, 1, ex]
            if pc and ex:
                en[pc] += 1
                eS[pc] += S
                eL[pc] += L
                hS[S] += 1
    r = acc.result()
    assert r["counts"].tolist() == exp.tolist()
    assert r["mem_n"].tolist() == en.tolist()
    assert r["mem_S"].tolist() == eS.tolist()
    assert r["mem_L"].tolist() == eL.tolist()
    assert r["hS"].tolist() == hS.tolist()
    assert r["PW_T"][0] == exp[1] and r["PW_W"][0] == exp[3]
    assert ev.invariants(r) == []


def test_single_event_definitions_against_sets():
    """32-lane random events: S/L equal numpy.unique sizes; counts equal bin().count."""
    rng = np.random.default_rng(7)
    n = 2000
    A = rng.integers(1, 2**32, size=n, dtype=np.uint64).astype(np.uint32)
    P = rng.integers(0, 2**32, size=n, dtype=np.uint64).astype(np.uint32)
    base = rng.integers(0, 2**40, size=(n, 1), dtype=np.uint64) & ~np.uint64(127)
    addr = base + rng.integers(0, 8192, size=(n, 32), dtype=np.uint64) * np.uint64(4)
    S, L = ev.sectors_lines(addr, A & P)
    for r in range(n):
        lanes = bits(int(A[r] & P[r]), 32)
        assert S[r] == len(np.unique(addr[r, lanes] >> np.uint64(5)))
        assert L[r] == len(np.unique(addr[r, lanes] >> np.uint64(7)))
    assert (ev.popc(A) == [bin(int(x)).count("1") for x in A]).all()


def test_listing8_fraction_identity():
    """C-5: Listing 8 adds 1/cnt per active thread (cnt = threads of the warp on my line);
    the sum is exactly the number of distinct lines, which the oracle counts as an integer."""
    g = json.load(open(os.path.join(GOLD, "listing8_example.json")))
    rng = np.random.default_rng(11)
    for trial in range(400):
        E = int(rng.integers(1, 2**32))
        lanes = bits(E, 32)
        addr = np.zeros((1, 32), dtype=np.uint64)
        addr[0] = rng.choice(ALPHABET + [8192, 8196, 8320], size=32)
        lines = [int(addr[0, l]) >> 7 for l in lanes]
        frac = sum(Fraction(1, lines.count(x)) for x in lines)
        _, L = ev.sectors_lines(addr, np.array([E], dtype=np.uint32))
        assert frac == L[0]
    # the paper's worked example: two threads on one line add 1/2 each -> one unique line
    addr = np.zeros((1, 32), dtype=np.uint64)
    addr[0, g["lanes"]] = g["addr"]
    E = sum(1 << l for l in g["lanes"])
    _, L = ev.sectors_lines(addr, np.array([E], dtype=np.uint32))
    assert Fraction(g["per_thread_increment"]) * len(g["lanes"]) == L[0] == g["unique_lines"]


def test_zero_active_mask_is_not_an_event():
    acc = ev.Accumulator(tiny_prog())
    acc.add(0, [0, 0], 0, [0, 1], [0xFFFFFFFF, 0])
    r = acc.result()
    assert r["counts"].tolist() == [1, 0, 1, 0]   # C-10: issued, not executed


def test_invariants_detect_a_dropped_term():
    acc = ev.Accumulator(tiny_prog())
    acc.add(0, [0], 1, [0xFF], [0xFF], np.arange(32, dtype=np.uint64)[None, :] * 64)
    r = acc.result()
    assert ev.invariants(r) == []
    r["H_t"][3] += 1
    assert "sum H = totals" in ev.invariants(r)


# ---------------------------------------------------------------- Ent_t at a guarded leader (A != E)
def guarded_leader_case():
    g = json.load(open(os.path.join(GOLD, "guarded_leader.json")))
    pr = g["program"]
    prog = {k: np.array(pr[k]) for k in ("opcode", "kind", "width", "bb", "is_leader", "guarded")}
    prog.update(n_pcs=4, n_opcodes=pr["n_opcodes"], n_bbs=2)
    evs = g["events"]
    base = 1 << 32
    addr = np.array([[base + 4 * l for l in range(32)] for _ in evs], dtype=np.uint64)
    cols = dict(pc=np.array([e["pc"] for e in evs]), A=np.array([int(e["A"], 16) for e in evs], dtype=np.uint32),
                P=np.array([int(e["P"], 16) for e in evs], dtype=np.uint32), addr=addr)
    return prog, cols, g["expect"]


def test_ent_t_counts_active_threads_at_a_guarded_leader():
    prog, c, exp = guarded_leader_case()
    acc = ev.Accumulator(prog)
    acc.add(0, np.zeros(len(c["pc"]), dtype=np.int64), c["pc"], c["A"], c["P"], c["addr"])
    r = acc.result()
    for k in ("Ent_t", "Ent_w", "Ins_t", "Ins_w", "counts"):
        assert r[k].tolist() == exp[k], k
    assert (r["mem_n"][0], r["mem_S"][0], r["mem_L"][0]) == (exp["mem_n0"], exp["mem_S0"], exp["mem_L0"])
    # I-5 with the guard corrections computed from the raw masks
    off_t = sum(bin(int(A) & ~int(P) & 0xFFFFFFFF).count("1") for pc, A, P in zip(c["pc"], c["A"], c["P"])
                if prog["guarded"][pc] and prog["bb"][pc] == 0)
    assert 3 * r["Ent_t"][0] - off_t == r["Ins_t"][0]
