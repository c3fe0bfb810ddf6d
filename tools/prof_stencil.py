"""Launch sequence for an ncu capture of the instrumented stencil (plain + BBCOUNT|MEMDIV)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_micro_villasnk19_b200 as pkg  # noqa: E402
from synth import uniform_f32  # noqa: E402

nb = pkg.nvbt
n = 8192
ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.BB | nb.MEMDIV)
x = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
y = torch.empty_like(x)
nb.nvbt_stencil(ctx, nb.TOOL_NONE, x, y, n)
nb.nvbt_stencil(ctx, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV, x, y, n)
nb.nvbt_stencil(ctx, nb.TOOL_BBCOUNT, x, y, n)
torch.cuda.synchronize()
