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
if which in ("all", "c5"):
    n = 1 << 26
    rctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    hdr = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty(n * 256, dtype=torch.uint8, device="cuda")
    nb.nvbt_gen_events(rctx, 0x4E5642544E564254, 0, n, hdr, addr)
    nb.nvbt_replay(rctx, hdr, addr, n)
    nb.nvbt_count(rctx)
torch.cuda.synchronize()
print("done")
