"""Pins for the F4 oracle (oracle/models/wfft.py; EVENT_MODEL §3.6, paper §6.3).

The DFT definition is pinned by a library routine (numpy.fft.fft), closed forms that a wrong sign, index
or normalisation would break (a single complex exponential maps to 32·δ at the right bin, constants to
32·δ_0), Parseval, Hermitian symmetry of real inputs and the inverse-DFT round trip. The event model is
pinned by hand-derived per-warp closed forms (EM §3.6: W_issued = 6 + 8k / 40 + 43k, W_exec = 4 + 8k /
38 + 43k for a warp with k transforms) and by the invariants of I-2."""
import numpy as np
import pytest

from oracle import events as ev, programs
from oracle.models import wfft

BASE = 1 << 32


def rand_c(shape, seed):
    r = np.random.default_rng(seed)
    return r.uniform(-1, 1, shape) + 1j * r.uniform(-1, 1, shape)


# ---------------------------------------------------------------- the transform
def test_dft_matches_numpy_fft():
    x = rand_c((64, 32), 11)
    assert np.allclose(wfft.dft32(x), np.fft.fft(x, axis=-1), rtol=0, atol=1e-12)


@pytest.mark.parametrize("m", [0, 1, 5, 16, 31])
def test_dft_single_exponential(m):
    n = np.arange(32)
    X = wfft.dft32(np.exp(2j * np.pi * m * n / 32))     # forward sign: energy lands in bin m, not 32 - m
    expect = np.zeros(32, dtype=complex)
    expect[m] = 32
    assert np.allclose(X, expect, atol=1e-12)


def test_dft_constant_and_delta():
    assert np.allclose(wfft.dft32(np.ones(32)), 32 * (np.arange(32) == 0), atol=1e-12)
    d = np.zeros(32); d[0] = 1
    assert np.allclose(wfft.dft32(d), np.ones(32), atol=1e-15)
    d = np.zeros(32); d[8] = 1                           # delayed delta: X[k] = (-i)^k
    assert np.allclose(wfft.dft32(d), (-1j) ** np.arange(32), atol=1e-12)


def test_dft_parseval_hermitian_inverse():
    x = rand_c((16, 32), 12)
    X = wfft.dft32(x)
    assert np.allclose((abs(X) ** 2).sum(1), 32 * (abs(x) ** 2).sum(1), rtol=1e-12)
    xr = x.real
    Xr = wfft.dft32(xr)
    k = np.arange(1, 32)
    assert np.allclose(Xr[:, 32 - k], np.conj(Xr[:, k]), atol=1e-12)
    # inverse DFT: x[n] = (1/32) Σ_k X[k] exp(+2πi nk/32) = conj(DFT(conj(X))) / 32
    assert np.allclose(np.conj(wfft.dft32(np.conj(X))) / 32, x, atol=1e-12)


def test_brev5():
    for l in range(32):
        assert wfft.brev5(l) == int(format(l, "05b")[::-1], 2)
    assert (wfft.brev5(wfft.brev5(np.arange(32))) == np.arange(32)).all()


# ---------------------------------------------------------------- the programs
def test_programs_shape():
    e, s = programs.wfft_emu(), programs.wfft_sw()
    assert e["n_pcs"] == 14 and s["n_pcs"] == 83
    assert e["opcode"][7] == programs.WFFT32 and (s["opcode"] != programs.WFFT32).all()
    assert (s["opcode"][41:77] == programs.SHFL).sum() == 10     # 2 shuffles per stage, 5 stages
    assert e["n_opcodes"] == s["n_opcodes"] == 32


# ---------------------------------------------------------------- events: per-warp closed forms
@pytest.mark.parametrize("variant", [wfft.EMU, wfft.SW])
@pytest.mark.parametrize("n_fft,ctas", [(1, 1), (8, 1), (21, 2), (100, 3), (5, 2)])
def test_events_closed_form(variant, n_fft, ctas):
    prog = programs.wfft_sw() if variant == wfft.SW else programs.wfft_emu()
    W = 8 * ctas
    acc = ev.Accumulator(prog, n_warps=W)
    wfft.run(acc, variant, n_fft, ctas, BASE, BASE + (1 << 24))
    r = acc.result()
    assert ev.invariants(r) == []
    body, pre_i, pre_e = (43, 40, 38) if variant == wfft.SW else (8, 6, 4)
    Wi = We = 0
    for w in range(W):
        k = len(range(w, n_fft, W))                      # transforms of warp w
        wi = pre_i + body * k if k else 5
        we = pre_e + body * k if k else 5         # idle warp: its EXIT executes
        assert r["PW_W"][w] == we, (w, k)
        assert r["PW_T"][w] == 32 * we                   # every executing lane is active
        Wi += wi
        We += we
    assert r["counts"].tolist() == [32 * Wi, 32 * We, Wi, We]
    # per-transform histogram entries
    if variant == wfft.EMU:
        assert r["H_w"][programs.WFFT32] == n_fft
    else:
        assert r["H_w"][programs.SHFL] == 10 * n_fft
        assert r["H_w"][programs.FMUL] == 8 * n_fft
        assert r["H_w"][programs.FFMA] == (4 * 4 + 2) * n_fft
    # divergence: each load/store covers one 256 B-aligned row: 8 sectors, 2 lines
    mem_pcs = (40, 78) if variant == wfft.SW else (6, 9)
    for pc in mem_pcs:
        assert r["mem_n"][pc] == n_fft and r["mem_S"][pc] == 8 * n_fft and r["mem_L"][pc] == 2 * n_fft
    assert r["hS"][8] == 2 * n_fft and r["hL"][2] == 2 * n_fft


def test_events_bb_identity():
    """I-5: Ins = len·Ent − Off per BB (the BB-entry mode's derivation) on the SW program."""
    prog = programs.wfft_sw()
    acc = ev.Accumulator(prog)
    wfft.run(acc, wfft.SW, 37, 2, BASE, BASE)
    r = acc.result()
    # BB2 (the loop): 43 pcs entered once per transform; the BRA is predicated off once per live warp
    live = min(37, 16)
    assert r["Ent_w"][2] == 37 and r["Ins_w"][2] == 43 * 37 - live
    assert r["Ent_w"][1] == live and r["Ins_w"][1] == 34 * live
