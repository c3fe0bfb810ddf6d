"""Launch sequence for an ncu capture of the C4 trace producer (8192^2 stencil, TOOL_TRACE, one iteration)
with the pinned channel: one plain launch, then one traced launch into a ring that holds all of its
12.6 M records (no consumer needed, so ncu's kernel replay never waits on the host)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_micro_villasnk19_b200 as pkg  # noqa: E402
from synth import uniform_f32  # noqa: E402

nb = pkg.nvbt
n = 8192
arg = sys.argv[1] if len(sys.argv) > 1 else ""
compact = {"compact": True, "line": 128}.get(arg, False)   # 176 B slots (EM 5.1) / 128 B line slots (EM 5.2)
ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.TRACE)
x = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
y = torch.empty_like(x)
records = 2 * (n * n // 32) + 4 * (n - 2) * (n // 32)
ring = torch.empty(nb.nvbt_channel_bytes(records + 4096, compact=compact), dtype=torch.uint8, pin_memory=True)
ch = nb.nvbt_channel_open(ctx, ring, compact=compact)
nb.nvbt_stencil(ctx, nb.TOOL_NONE, x, y, n)
nb.nvbt_stencil(ctx, nb.TOOL_TRACE, x, y, n)
torch.cuda.synchronize()
print("dropped", nb.nvbt_channel_dropped(ch), "records", records)
