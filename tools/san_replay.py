"""Small staged + single-pass replay for compute-sanitizer runs (racecheck / synccheck / initcheck):
`compute-sanitizer --tool racecheck python tools/san_replay.py [n_events]`. The generated stream holds all
six address patterns, so every pass-B path (scan, window tags, wide-row hash + resolve, bitonic fallback)
runs; prints the counts so a run can be compared with an unsanitised one."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_micro_villasnk19_b200 as pkg  # noqa: E402

nb, dr = pkg.nvbt, pkg.drivers
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 14
hdr = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
addr = torch.empty(n * 256, dtype=torch.uint8, device="cuda")
out = []
for staged in (True, False):
    ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)
    nb.nvbt_gen_events(ctx, 0x4E5642544E564254, 0, n, hdr, addr)
    if staged:
        scratch = torch.empty(nb.nvbt_replay_scratch_size(ctx, n), dtype=torch.uint8, device="cuda")
        nb.nvbt_replay_staged(ctx, hdr, addr, n, scratch)
    else:
        nb.nvbt_replay(ctx, hdr, addr, n)
    per, tot, hs, hl = nb.nvbt_mem_divergence(ctx)
    out.append((tuple(int(x) for x in nb.nvbt_count(ctx)), tuple(int(x) for x in tot), tuple(int(x) for x in hs)))
print("staged", out[0])
print("single", out[1])
assert out[0] == out[1], "staged and single-pass replay disagree"
print("ok")
