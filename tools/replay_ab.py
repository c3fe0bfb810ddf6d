"""A/B timing of the staged replay (C5's bench path) across library builds.

usage: python tools/replay_ab.py lib1.so [lib2.so ...]   (each timed in its own subprocess via NVBT_LIB)
Prints, per library, the median of 10 timed calls on one 2^27-event chunk (CUDA events), the per-pass
kernel times (k_rpA / k_rpB, torch.profiler-free: two separate timed calls with MEMDIV off/on), and a
checksum of the accumulators so the variants can be seen to agree."""
import json
import os
import subprocess
import sys

CHILD = r'''
import json, statistics, sys, torch
sys.path.insert(0, "@ROOT@")
import paper_conf_micro_villasnk19_b200 as pkg
nb = pkg.nvbt
n = 1 << 27
hdr = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
addr = torch.empty(n * 256, dtype=torch.uint8, device="cuda")
res = {}
for name, flags in (("A_only", nb.COUNT | nb.OPHIST | nb.BB), ("A+B", nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)):
    ctx = nb.nvbt_init(nb.W_REPLAY, flags)
    scratch = torch.empty(nb.nvbt_replay_scratch_size(ctx, n), dtype=torch.uint8, device="cuda")
    nb.nvbt_gen_events(ctx, 0x4E5642544E564254, 0, n, hdr, addr)
    for _ in range(3):
        nb.nvbt_replay_staged(ctx, hdr, addr, n, scratch)
    ts = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); nb.nvbt_replay_staged(ctx, hdr, addr, n, scratch); e1.record(); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    acc = nb.nvbt_accum_view(ctx)
    res[name] = {"ms": statistics.median(ts), "min_ms": min(ts), "checksum": int((acc * torch.arange(1, acc.numel() + 1, device="cuda")).sum().item())}
_, tot, _, _ = nb.nvbt_mem_divergence(ctx)
mem = int(tot[0]) // 13
res["events_per_s"] = n / (res["A+B"]["ms"] / 1e3)
res["hbm_frac"] = (16 * n + 256 * mem) / (res["A+B"]["ms"] / 1e3) / 6.552e12
res["passB_ms_est"] = res["A+B"]["ms"] - res["A_only"]["ms"]
print("RESULT " + json.dumps(res))
'''

root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for lib in sys.argv[1:]:
    env = dict(os.environ, NVBT_LIB=os.path.abspath(lib))
    r = subprocess.run([sys.executable, "-c", CHILD.replace("@ROOT@", root)], capture_output=True, text=True, env=env)
    line = [l for l in r.stdout.splitlines() if l.startswith("RESULT ")]
    print(os.path.basename(lib), line[0][7:] if line else r.stderr[-2000:], flush=True)
