"""GPU parity for F4, instruction emulation (EVENT_MODEL §3.6; paper §6.3).

Events (counts, opcode/BB histograms, per-warp counts, divergence, trace records) are integer and compared
bit-exactly with oracle/models/wfft.py. Transform values are fp32 on the GPU and compared with the fp64 DFT
definition (oracle `dft32`) under the radix-2 FFT error bound derived in DESIGN.md (F4):
‖X̂ − X‖₂ ≤ log2(32) · η · ‖X‖₂ with η ≤ 8u (u = 2^-24: twiddle error + one complex multiply-add per
stage), i.e. 40u per transform. The emulated (proxy + NVBT_TOOL_EMU) and the software kernel compute the
transform with the same operations, so their outputs must be bit-identical."""
import numpy as np
import pytest

from oracle import events as ev, programs, trace
from oracle.models import wfft as m_wf
from synth import uniform_f32

from .gpu_util import read_all, assert_same, gpu_invariants

pytestmark = pytest.mark.gpu

COUNT_KEYS = ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t"]
MEM_KEYS = ["mem_n", "mem_S", "mem_L", "hS", "hL"]
REL_BOUND = 40 * 2.0 ** -24


def inputs(n_fft, seed=5):
    """complex64 [n_fft, 32], re and im ~ U[-1, 1) (numpy PCG64 for test sizes, torch's CUDA generator for
    the full bench size)."""
    import torch
    if n_fft <= 1 << 16:
        x = uniform_f32((n_fft, 32, 2), seed, -1, 1)
        xt = torch.from_numpy(x).cuda().view(torch.complex64).reshape(n_fft, 32)
    else:
        g = torch.Generator(device="cuda").manual_seed(seed)
        xt = (torch.rand((n_fft, 32, 2), generator=g, device="cuda") * 2 - 1).view(torch.complex64).reshape(n_fft, 32)
    return xt, torch.zeros_like(xt)


def tools_of(nb, names):
    t = 0
    for n in names.split("|"):
        if n:
            t |= getattr(nb, "TOOL_" + n)
    return t


def check_values(x, X):
    ref = m_wf.dft32(x.cpu().numpy().astype(np.complex128))
    got = X.cpu().numpy().astype(np.complex128)
    err = np.linalg.norm(got - ref, axis=1)
    bound = REL_BOUND * np.linalg.norm(ref, axis=1) + 1e-30
    assert (err <= bound).all(), f"max rel err {np.max(err / np.linalg.norm(ref, axis=1)) / 2**-24:.2f} u"


@pytest.mark.parametrize("n_fft,ctas", [(1, 1), (100, 3), (1000, 7), (4099, 37), (5, 2)])
@pytest.mark.parametrize("variant,tools", [("PROXY", "EMU|COUNT|MEMDIV"), ("PROXY", "EMU|BBCOUNT|MEMDIV"),
                                           ("PROXY", "COUNT"), ("SOFTWARE", "COUNT|MEMDIV"),
                                           ("SOFTWARE", "BBCOUNT|MEMDIV"), ("SOFTWARE", "MEMDIV")])
def test_wfft_parity(nvbt, n_fft, ctas, variant, tools):
    nb = nvbt.nvbt
    v = getattr(nb, "WFFT_" + variant)
    w = nb.W_WFFT_EMU if v == nb.WFFT_PROXY else nb.W_WFFT_SW
    nw = nb.nvbt_workload_warps(w, n_fft, ctas)
    ctx = nb.nvbt_init(w, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
    x, X = inputs(n_fft)
    t = tools_of(nb, tools)
    nb.nvbt_wfft32(ctx, t, v, x, X, n_fft, ctas)
    g = read_all(nb, ctx, per_warp=True)
    prog = programs.wfft_emu() if v == nb.WFFT_PROXY else programs.wfft_sw()
    acc = ev.Accumulator(prog, n_warps=nw)
    m_wf.run(acc, m_wf.EMU if v == nb.WFFT_PROXY else m_wf.SW, n_fft, ctas, x.data_ptr(), X.data_ptr())
    r = acc.result()
    keys = (COUNT_KEYS + ["PW_T", "PW_W"] if ("COUNT" in tools) else []) + (MEM_KEYS if "MEMDIV" in tools else [])
    assert_same(g, r, keys, f"wfft {variant} {tools} n_fft={n_fft} ctas={ctas}")
    if "COUNT" in tools:
        gpu_invariants(g)
    if v == nb.WFFT_PROXY and not (t & nb.TOOL_EMU):
        import torch
        assert torch.equal(X, x)                       # native proxy: a register move
    else:
        check_values(x, X)


def test_emulated_equals_software_bitwise(nvbt):
    """wfft32emu() is functionally the software transform: identical fp32 bits, with and without hooks."""
    import torch
    nb = nvbt.nvbt
    n_fft = 3001
    x, X1 = inputs(n_fft, seed=6)
    X2, X3 = torch.zeros_like(X1), torch.zeros_like(X1)
    nb.nvbt_wfft32(None, nb.TOOL_EMU, nb.WFFT_PROXY, x, X1, n_fft, 5)
    nb.nvbt_wfft32(None, nb.TOOL_NONE, nb.WFFT_SOFTWARE, x, X2, n_fft, 9)
    ctx = nb.nvbt_init(nb.W_WFFT_SW, nb.COUNT)
    nb.nvbt_wfft32(ctx, nb.TOOL_COUNT, nb.WFFT_SOFTWARE, x, X3, n_fft, 2)
    torch.cuda.synchronize()
    assert torch.equal(X1.view(torch.int64), X2.view(torch.int64))
    assert torch.equal(X1.view(torch.int64), X3.view(torch.int64))
    check_values(x, X1)


def test_wfft_special_inputs(nvbt):
    """Closed forms through the GPU path: delta -> ones, constant -> 32 delta_0, single exponential -> 32 delta_m."""
    import torch
    nb = nvbt.nvbt
    n = np.arange(32)
    rows = [np.eye(32)[0], np.ones(32), np.exp(2j * np.pi * 5 * n / 32), np.exp(2j * np.pi * 31 * n / 32)]
    x = torch.from_numpy(np.array(rows, dtype=np.complex64)).cuda()
    X = torch.zeros_like(x)
    nb.nvbt_wfft32(None, nb.TOOL_EMU, nb.WFFT_PROXY, x, X, len(rows), 1)
    got = X.cpu().numpy()
    exp = np.zeros((4, 32), dtype=complex)
    exp[0] = 1
    exp[1, 0] = 32
    exp[2, 5] = 32
    exp[3, 31] = 32
    assert np.abs(got - exp).max() < 32 * 40 * 2.0 ** -24


def test_wfft_bench_config_sampled(nvbt):
    """The launch configuration bench.py times (n_fft = 2^24, one resident wave of CTAs): closed-form
    totals, the oracle's events on sampled warps (PER_WARP) and sampled transforms against the DFT."""
    import torch
    nb = nvbt.nvbt
    n_fft = 1 << 24
    x, X = inputs(n_fft, seed=7)
    cases = [(v, w, body, pre_i, pre_e, ct | (nb.TOOL_EMU if v == nb.WFFT_PROXY else 0))
             for v, w, body, pre_i, pre_e in ((nb.WFFT_PROXY, nb.W_WFFT_EMU, 8, 6, 4),
                                              (nb.WFFT_SOFTWARE, nb.W_WFFT_SW, 43, 40, 38))
             for ct in (nb.TOOL_COUNT, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV)]
    for v, w, body, pre_i, pre_e, t in cases:       # EMU|COUNT is the bench's timed launch
        ctas = nb.nvbt_wfft32_max_ctas(t, v)
        assert ctas % 148 == 0
        W = 8 * ctas
        ctx = nb.nvbt_init(w, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=W)
        X.zero_()
        nb.nvbt_wfft32(ctx, t, v, x, X, n_fft, ctas)
        g = read_all(nb, ctx, per_warp=True)
        k = np.array([len(range(i, n_fft, W)) for i in range(W)])
        assert g["counts"][2] == (pre_i + body * k).sum() and g["counts"][3] == (pre_e + body * k).sum()
        assert g["counts"][1] == 32 * g["counts"][3]
        sample = np.array([0, 1, 7, 8, W // 3, W // 2, W - 1])
        acc = ev.Accumulator(programs.wfft_emu() if v == nb.WFFT_PROXY else programs.wfft_sw(), n_warps=W)
        m_wf.run(acc, m_wf.EMU if v == nb.WFFT_PROXY else m_wf.SW, n_fft, ctas, x.data_ptr(), X.data_ptr(),
                 warps=sample)
        r = acc.result()
        assert (g["PW_W"][sample] == r["PW_W"][sample]).all() and (g["PW_T"][sample] == r["PW_T"][sample]).all()
        if t & nb.TOOL_MEMDIV:
            mem_pcs = [6, 9] if v == nb.WFFT_PROXY else [40, 78]
            assert (g["mem_n"][mem_pcs] == n_fft).all() and (g["mem_S"][mem_pcs] == 8 * n_fft).all()
            assert (g["mem_L"][mem_pcs] == 2 * n_fft).all()
        rows = torch.tensor([0, 1, 12345, n_fft // 2, n_fft - 2, n_fft - 1], device="cuda")
        check_values(x[rows], X[rows])
        gpu_invariants(g)


def test_wfft_trace_records(nvbt):
    """TRACE on the emulated kernel: the record multiset equals the oracle's (EM §5)."""
    import torch
    nb = nvbt.nvbt
    n_fft, ctas = 333, 4
    ctx = nb.nvbt_init(nb.W_WFFT_EMU, nb.COUNT | nb.TRACE)
    ring = torch.empty(nb.nvbt_channel_bytes(4096), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring)
    x, X = inputs(n_fft, seed=8)
    nb.nvbt_wfft32(ctx, nb.TOOL_EMU | nb.TOOL_TRACE | nb.TOOL_COUNT, nb.WFFT_PROXY, x, X, n_fft, ctas)
    acc = ev.Accumulator(programs.wfft_emu(), trace=True, keep_records=True)
    m_wf.run(acc, m_wf.EMU, n_fft, ctas, x.data_ptr(), X.data_ptr())
    exp = acc.record_array()
    dst = np.zeros((len(exp) + 1024, 288), dtype=np.uint8)
    got_n = nb.nvbt_channel_drain_copy(ch, dst, timeout_us=60_000_000)
    assert got_n == len(exp) == 2 * n_fft
    assert (trace.sort_records(dst[:got_n]) == trace.sort_records(exp)).all()
    check_values(x, X)


def test_wfft_edge_cases_and_errors(nvbt):
    import torch
    nb = nvbt.nvbt
    ctx = nb.nvbt_init(nb.W_WFFT_SW, nb.COUNT)
    x, X = inputs(64)
    nb.nvbt_wfft32(ctx, nb.TOOL_COUNT, nb.WFFT_SOFTWARE, x, X, 0, 3)      # empty: nothing launched
    assert (nb.nvbt_count(ctx) == 0).all()
    for bad in (
        lambda: nb.nvbt_wfft32(ctx, nb.TOOL_EMU, nb.WFFT_SOFTWARE, x, X, 64, 1),     # no proxy to emulate
        lambda: nb.nvbt_wfft32(ctx, nb.TOOL_COUNT, nb.WFFT_PROXY, x, X, 64, 1),      # wrong program
        lambda: nb.nvbt_wfft32(None, 0, nb.WFFT_PROXY, x, x, 64, 1),                 # in place
        lambda: nb.nvbt_wfft32(None, 0, nb.WFFT_PROXY, x, X, 64, 0),                 # no CTAs
        lambda: nb.nvbt_wfft32(None, 0, 7, x, X, 64, 1),                             # bad variant
        lambda: nb.nvbt_wfft32(None, nb.TOOL_COUNT, nb.WFFT_PROXY, x, X, 64, 1),     # counting without ctx
    ):
        with pytest.raises(nb.NvbtError):
            bad()
    # more CTAs than transforms: idle warps issue and execute pcs 0-4 only
    ctx2 = nb.nvbt_init(nb.W_WFFT_EMU, nb.COUNT | nb.PER_WARP, n_warps=8 * 9)
    nb.nvbt_wfft32(ctx2, nb.TOOL_COUNT | nb.TOOL_EMU, nb.WFFT_PROXY, x, X, 3, 9)
    c, pwt, pww = nb.nvbt_count(ctx2, per_warp=True)
    assert pww.tolist() == [12] * 3 + [5] * 69
    torch.cuda.synchronize()
