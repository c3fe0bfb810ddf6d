"""Exactness of the privatised counters past 2^32: per-site counters live in u32
registers and CTA shared bins before the 64-bit global flush, so long loops must spill them before they
can wrap (nvbt_hooks.cuh Hooks::tick, every 2^16 loop instances). SGEMM with M = 32, N = 8 (one CTA, 8
warps) and K = 2^25 + 3: every warp runs 6K + 12 > 2 x 10^8 warp instructions, its executed-thread count
32 (6K + 10) > 2^32, and the CTA's A-load sector sum 8 x 32K > 2^32. All results equal the closed form
(EM §3.2) and the C oracle exactly."""
import numpy as np
import pytest

from oracle import coracle as co, programs

from .gpu_util import read_all, assert_same

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.mark.parametrize("tools", ["COUNT|MEMDIV", "BBCOUNT|MEMDIV"])
def test_sgemm_k_beyond_u32(nvbt, tools):
    import torch
    nb = nvbt.nvbt
    M, N, K = 32, 8, (1 << 25) + 3
    t = 0
    for x in tools.split("|"):
        t |= getattr(nb, "TOOL_" + x)
    W = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
    assert W == 8
    ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=W)
    A = torch.ones(M, K, device="cuda")
    B = torch.ones(K, N, device="cuda")
    Cm = torch.empty(M, N, device="cuda")
    nb.nvbt_sgemm(ctx, t, A, B, Cm, M, N, K)
    g = read_all(nb, ctx, per_warp=True)
    # closed form (EM §3.2): no lane exits (pc 7 issued, never executed); the last BRA is predicated off
    wi = 12 + 6 * K
    we = wi - 2
    assert g["counts"].tolist() == [32 * W * wi, 32 * W * we, W * wi, W * we]
    assert g["PW_T"].tolist() == [32 * we] * W and g["PW_W"].tolist() == [we] * W
    assert 32 * we > 1 << 32
    # divergence: A rows 4K bytes apart (32 lines), B a broadcast (1, 1), C 32 B apart (32 sectors, 8 lines)
    assert (g["mem_n"][10], g["mem_S"][10], g["mem_L"][10]) == (W * K, 32 * W * K, 32 * W * K)
    assert (g["mem_n"][11], g["mem_S"][11], g["mem_L"][11]) == (W * K, W * K, W * K)
    assert (g["mem_n"][16], g["mem_S"][16], g["mem_L"][16]) == (W, 32 * W, 8 * W)
    assert g["hS"][32] == W * K + W and g["hS"][1] == W * K and g["hL"][8] == W
    r = co.sgemm(programs.sgemm(), M, N, K, A.data_ptr(), B.data_ptr(), Cm.data_ptr(), per_warp=True)
    assert_same(g, r, ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t", "mem_n", "mem_S", "mem_L",
                       "hS", "hL", "PW_T", "PW_W"], f"SGEMM K = 2^25 + 3 {tools}")
    # fp32 accumulation of K ones saturates at 2^24 (2^24 + 1 rounds to even): the computed product
    assert torch.all(Cm == float(1 << 24))


def test_bfs_hub_of_degree_2_24_is_reported(nvbt):
    """BFS keeps its edge-loop counters in u32 registers / CTA bins (no spill code: it would cost the
    latency-bound BFS occupancy), exact while every warp's degree is < 2^24. A star with 2^24 leaves is
    flagged on the device and the read call fails loudly (NVBT_EINVAL) instead of returning wrapped
    counts; nvbt_reset clears the flag."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n = (1 << 24) + 1
    rowptr = np.empty(n + 1, dtype=np.int32)  # vertex 0: edges to 1 .. 2^24; every leaf: one edge back to 0
    rowptr[0] = 0
    rowptr[1] = 1 << 24
    rowptr[2:] = (1 << 24) + np.arange(1, n, dtype=np.int64)
    col = np.concatenate([np.arange(1, n, dtype=np.int32), np.zeros(n - 1, dtype=np.int32)])
    rp, cl = torch.from_numpy(rowptr).cuda(), torch.from_numpy(col).cuda()
    ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    cost, levels = dr.run_bfs(ctx, nb.TOOL_BBCOUNT, rp, cl, 0)
    assert levels == 2 and int(cost.max()) == 1
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_count(ctx)
    assert e.value.code == nb.EINVAL
    nb.nvbt_reset(ctx)
    assert (nb.nvbt_count(ctx) == 0).all()


def test_wfft_loop_beyond_spill_chunk(nvbt):
    """WFFT32's per-warp transform loop runs in chunks of 2^20 instances with the counters spilled to the
    64-bit bins in between (Hooks::spill): one CTA (8 warps), k_w = 2^20 + 2 transforms per warp. Counts and
    per-warp arrays equal the EM §3.6 closed form (W_issued = 6 + 8 k_w, W_exec = 4 + 8 k_w per warp for
    WFFT_EMU), divergence bins too (each load / store: 256 contiguous bytes = 8 sectors, 2 lines)."""
    import torch
    nb = nvbt.nvbt
    ctas, kw = 1, (1 << 20) + 2
    W = 8 * ctas
    n_fft = W * kw
    x = torch.zeros((n_fft, 32, 2), dtype=torch.float32, device="cuda").view(torch.complex64).reshape(n_fft, 32)
    X = torch.empty_like(x)
    ctx = nb.nvbt_init(nb.W_WFFT_EMU, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=W)
    nb.nvbt_wfft32(ctx, nb.TOOL_EMU | nb.TOOL_COUNT | nb.TOOL_MEMDIV, nb.WFFT_PROXY, x, X, n_fft, ctas)
    g = read_all(nb, ctx, per_warp=True)
    wi, we = 6 + 8 * kw, 4 + 8 * kw
    assert g["counts"].tolist() == [32 * W * wi, 32 * W * we, W * wi, W * we]
    assert g["PW_T"].tolist() == [32 * we] * W and g["PW_W"].tolist() == [we] * W
    assert (g["mem_n"][6], g["mem_S"][6], g["mem_L"][6]) == (W * kw, 8 * W * kw, 2 * W * kw)
    assert (g["mem_n"][9], g["mem_S"][9], g["mem_L"][9]) == (W * kw, 8 * W * kw, 2 * W * kw)
    assert g["hS"][8] == 2 * W * kw and g["hL"][2] == 2 * W * kw
    del x, X
    torch.cuda.empty_cache()
