"""Hypothesis property tests of the oracle's per-event functions on random 32-lane events (SURVEY §4 plan
item 1; invariants of SURVEY §8(c) I-2). Each property is a fact of the definitions in EM §2 that a
plausible slip would break: a dropped lane, a wrong shift, E taken as A, a sector/line mix-up."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import events as ev, programs

FULL = 0xFFFFFFFF
masks = st.integers(min_value=0, max_value=FULL)
# addresses: a random 40-bit base plus lane offsets drawn from a few scales (same word, window, wide)
scales = st.sampled_from([4, 32, 128, 1 << 12, 1 << 20, 1 << 38])


@st.composite
def events(draw):
    A = draw(masks)
    P = draw(masks)
    base = draw(st.integers(min_value=0, max_value=(1 << 40) - 1))
    scale = draw(scales)
    offs = draw(st.lists(st.integers(min_value=0, max_value=scale - 1), min_size=32, max_size=32))
    width = draw(st.sampled_from([1, 2, 4, 8, 16]))
    addr = [((base + o) // width) * width for o in offs]
    return A, P, addr


def one(A, P, addr):
    S, L = ev.sectors_lines(np.array([addr], dtype=np.uint64), np.array([A & P], dtype=np.uint32))
    return int(S[0]), int(L[0])


@settings(max_examples=300, deadline=None)
@given(events())
def test_sectors_lines_bounds(e):
    """E != 0: 1 <= L <= S <= min(32, 4L) and S <= |E|; E == 0: S = L = 0."""
    A, P, addr = e
    S, L = one(A, P, addr)
    n = bin(A & P).count("1")
    if n == 0:
        assert S == L == 0
    else:
        assert 1 <= L <= S <= min(n, 32) and S <= 4 * L


@settings(max_examples=300, deadline=None)
@given(events())
def test_sectors_lines_only_lanes_of_E(e):
    """Changing the address of a lane outside E never changes S or L; a lane inside E can."""
    A, P, addr = e
    E = A & P
    S, L = one(A, P, addr)
    for l in range(32):
        if not (E >> l) & 1:
            moved = list(addr)
            moved[l] = (addr[l] + (1 << 30)) % (1 << 48)
            assert one(A, P, moved) == (S, L)


@settings(max_examples=200, deadline=None)
@given(events(), st.permutations(list(range(32))))
def test_sectors_lines_order_free(e, perm):
    """S and L are set sizes: permuting lanes together with their mask bits changes nothing."""
    A, P, addr = e
    E = A & P
    pE = sum(((E >> perm[l]) & 1) << l for l in range(32))
    paddr = [addr[perm[l]] for l in range(32)]
    assert one(pE, FULL, paddr) == one(A, P, addr)


@settings(max_examples=200, deadline=None)
@given(events())
def test_sectors_lines_match_sets(e):
    """Against the set definition written out (Python ints, no numpy)."""
    A, P, addr = e
    E = A & P
    lanes = [l for l in range(32) if (E >> l) & 1]
    assert one(A, P, addr) == (len({addr[l] >> 5 for l in lanes}), len({addr[l] >> 7 for l in lanes}))


@settings(max_examples=100, deadline=None)
@given(st.lists(events(), min_size=1, max_size=40), st.data())
def test_accumulator_invariants_and_additivity(evs, data):
    """I-2 invariants hold for any batch of replay-program events, and splitting the batch into two
    accumulators that are then summed gives the single accumulator's result (EM §4 additivity)."""
    prog = programs.replay()
    mem = np.nonzero(programs.is_mem(prog))[0]
    n = len(evs)
    pcs = np.array([int(mem[data.draw(st.integers(0, len(mem) - 1))]) if data.draw(st.booleans())
                    else data.draw(st.integers(0, prog["n_pcs"] - 1)) for _ in range(n)], dtype=np.int64)
    A = np.array([max(a, 1) for a, _, _ in evs], dtype=np.uint32)
    P = np.array([p for _, p, _ in evs], dtype=np.uint32)
    addr = np.array([x for _, _, x in evs], dtype=np.uint64)
    warp = np.zeros(n, dtype=np.int64)
    whole = ev.Accumulator(prog)
    whole.add(0, warp, pcs, A, P, addr)
    r = whole.result()
    assert ev.invariants(r) == []
    k = data.draw(st.integers(0, n))
    a, b = ev.Accumulator(prog), ev.Accumulator(prog)
    a.add(0, warp[:k], pcs[:k], A[:k], P[:k], addr[:k])
    b.add(0, warp[k:], pcs[k:], A[k:], P[k:], addr[k:])
    ra, rb = a.result(), b.result()
    for key, v in r.items():
        if isinstance(v, np.ndarray):
            assert np.array_equal(v, ra[key] + rb[key]), key


if __name__ == "__main__":
    pytest.main([__file__, "-q"])
