"""Minimal launch sequence for ncu captures: one plain and one instrumented launch of each bench
workload (no timing; numbers printed under a profiler are never bench values)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_micro_villasnk19_b200 as pkg  # noqa: E402
from synth import uniform_f32  # noqa: E402

nb, dr = pkg.nvbt, pkg.drivers
which = sys.argv[1] if len(sys.argv) > 1 else "all"
if which in ("all", "c2"):
    M = N = K = 1024
    ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.BB | nb.MEMDIV)
    A = torch.from_numpy(uniform_f32((M, K), 3, -1, 1)).cuda()
    B = torch.from_numpy(uniform_f32((K, N), 4, -1, 1)).cuda()
    C = torch.empty(M, N, device="cuda")
    nb.nvbt_sgemm(ctx, nb.TOOL_NONE, A, B, C, M, N, K)
    nb.nvbt_sgemm(ctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV, A, B, C, M, N, K)
    nb.nvbt_sgemm(ctx, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV, A, B, C, M, N, K)
    nb.nvbt_count(ctx)
if which in ("all", "c1"):
    from synth import uniform_f32 as _u
    N = 65536
    c1 = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.OPHIST)
    a, b = torch.from_numpy(_u(N, 1)).cuda(), torch.from_numpy(_u(N, 2)).cuda()
    c = torch.empty_like(a)
    c1b = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.OPHIST | nb.BB)
    for _ in range(3):
        nb.nvbt_vectoradd(c1, nb.TOOL_NONE, a, b, c, N)
        nb.nvbt_vectoradd(c1, nb.TOOL_COUNT, a, b, c, N)
        nb.nvbt_vectoradd(c1b, nb.TOOL_BBCOUNT, a, b, c, N)
    nb.nvbt_count(c1)
if which == "f2":   # traced stencil into an HBM ring (F2 producer), 8192^2 x 2 launches, then the consumer
    from synth import uniform_f32 as _u
    n, iters = 8192, 2
    fctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.TRACE)
    x0 = torch.from_numpy(_u((n, n), 4)).cuda()
    b0, b1 = x0.clone(), torch.empty_like(x0)
    cap = iters * (2 * (n * n // 32) + 4 * (n - 2) * (n // 32))
    cap += cap // 50 + 148 * 4096
    ring = torch.zeros(64 + 288 * cap, dtype=torch.uint8, device="cuda")
    ch = nb.nvbt_channel_open(fctx, ring)
    dr.run_stencil(fctx, nb.TOOL_NONE, b0, b1, n, iters)
    dr.run_stencil(fctx, nb.TOOL_TRACE, b0, b1, n, iters)
    torch.cuda.synchronize()
if which in ("all", "c5"):
    n = 1 << 26
    rctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    hdr = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty(n * 256, dtype=torch.uint8, device="cuda")
    nb.nvbt_gen_events(rctx, 0x4E5642544E564254, 0, n, hdr, addr)
    if os.environ.get("NVBT_PROF_SINGLE"):
        nb.nvbt_replay(rctx, hdr, addr, n)
    else:   # staged two-pass replay (the bench default)
        scratch = torch.empty(nb.nvbt_replay_scratch_size(rctx, n), dtype=torch.uint8, device="cuda")
        nb.nvbt_replay_staged(rctx, hdr, addr, n, scratch)
    nb.nvbt_count(rctx)
if which in ("all", "f4"):
    n_fft = 1 << 24
    x = (torch.rand((n_fft, 32, 2), device="cuda") * 2 - 1).view(torch.complex64).reshape(n_fft, 32)
    X = torch.empty_like(x)
    ce = nb.nvbt_init(nb.W_WFFT_EMU, nb.COUNT | nb.BB | nb.MEMDIV)
    cs = nb.nvbt_init(nb.W_WFFT_SW, nb.COUNT | nb.BB | nb.MEMDIV)
    # bench head (EMU|COUNT) first, then the other bench modes
    for ctx, v, t in ((ce, nb.WFFT_PROXY, nb.TOOL_EMU | nb.TOOL_COUNT), (ce, nb.WFFT_PROXY, nb.TOOL_NONE),
                      (cs, nb.WFFT_SOFTWARE, nb.TOOL_NONE), (ce, nb.WFFT_PROXY, nb.TOOL_EMU),
                      (cs, nb.WFFT_SOFTWARE, nb.TOOL_COUNT),
                      (ce, nb.WFFT_PROXY, nb.TOOL_EMU | nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV)):
        nb.nvbt_wfft32(ctx, t, v, x, X, n_fft, nb.nvbt_wfft32_max_ctas(t, v))
    nb.nvbt_count(ce)
torch.cuda.synchronize()
print("done")
