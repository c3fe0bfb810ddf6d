"""Time the C2 SGEMM under each tool combination (CUDA events, L2 flushed between launches)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_micro_villasnk19_b200 as pkg  # noqa: E402
from synth import uniform_f32  # noqa: E402

nb = pkg.nvbt
M = N = K = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.BB | nb.MEMDIV)
A = torch.from_numpy(uniform_f32((M, K), 3, -1, 1)).cuda()
B = torch.from_numpy(uniform_f32((K, N), 4, -1, 1)).cuda()
C = torch.empty(M, N, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
out = {}
for name, t in [("plain", 0), ("COUNT", 1), ("BBCOUNT", 2), ("MEMDIV", 4), ("COUNT|MEMDIV", 5), ("BBCOUNT|MEMDIV", 6)]:
    ts = []
    for i in range(13):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        nb.nvbt_sgemm(ctx, t, A, B, C, M, N, K)
        e1.record()
        e1.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1))
    out[name] = sorted(ts)[len(ts) // 2]
print(json.dumps(out))
