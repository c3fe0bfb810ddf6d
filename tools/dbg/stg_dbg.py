import sys, torch
sys.path.insert(0, '.')
import paper_conf_micro_villasnk19_b200 as pkg
nb = pkg.nvbt
ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
n = 4096
hdr = torch.empty(n * 16, dtype=torch.uint8, device="cuda")
addr = torch.empty(n * 256, dtype=torch.uint8, device="cuda")
nb.nvbt_gen_events(ctx, 0x4E5642544E564254, 0, n, hdr, addr)
scratch = torch.empty(nb.nvbt_replay_scratch_size(ctx, n), dtype=torch.uint8, device="cuda")
print("scratch", scratch.numel())
nb.nvbt_replay_staged(ctx, hdr, addr, n, scratch)
torch.cuda.synchronize()
print(nb.nvbt_count(ctx))
