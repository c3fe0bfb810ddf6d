"""Host-side drivers of the synthetic workloads and the multi-GPU merge.

Everything here is orchestration: it enqueues library kernels on the context's stream and moves a few
scalars (the BFS `over` flag). No event arithmetic happens in Python.
"""
from __future__ import annotations



def _nb():
    from . import nvbt
    return nvbt


def shard_range(n: int, rank: int, world: int):
    """Contiguous [lo, hi) share of n units for `rank` of `world` (event ranges for C5)."""
    lo = n * rank // world
    hi = n * (rank + 1) // world
    return lo, hi


def bfs_buffers(n, device):
    import torch
    return {
        "mask": torch.zeros(n, dtype=torch.uint8, device=device),
        "visited": torch.zeros(n, dtype=torch.uint8, device=device),
        "updating": torch.zeros(n, dtype=torch.uint8, device=device),
        "cost": torch.full((n,), -1, dtype=torch.int32, device=device),
        "over": torch.zeros(1, dtype=torch.int32, device=device),
    }


def run_bfs(ctx, tools, rowptr, col, src, bufs=None, stream=None, max_levels=1 << 20):
    """Level-synchronous BFS of EM §3.3 from `src` (rowptr/col: int32 CUDA tensors).

    Returns (cost tensor, levels, over_host_list)."""
    import torch
    n = rowptr.numel() - 1
    b = bfs_buffers(n, rowptr.device) if bufs is None else bufs
    b["mask"].zero_(); b["visited"].zero_(); b["updating"].zero_(); b["cost"].fill_(-1)
    b["mask"][src] = 1
    b["visited"][src] = 1
    b["cost"][src] = 0
    over_h = torch.zeros(1, dtype=torch.int32, pin_memory=True)
    level = 0
    while level < max_levels:
        b["over"].zero_()
        b["updating"].zero_()
        _nb().nvbt_bfs_level(ctx, tools, rowptr, col, n, b["mask"], b["visited"], b["updating"], b["cost"],
                          b["over"], level, stream=stream)
        over_h.copy_(b["over"], non_blocking=True)
        torch.cuda.current_stream().synchronize() if ctx is None else _sync(ctx)
        level += 1
        if int(over_h[0]) == 0:
            break
    return b["cost"], level


def _sync(ctx):
    import torch
    s = ctx.stream if ctx.stream is not None else torch.cuda.current_stream(ctx.device)
    s.synchronize()


def run_stencil(ctx, tools, buf0, buf1, n, iters, stream=None):
    """Iteration it reads buffer it % 2 and writes (it + 1) % 2 (EM §3.4). Returns the final buffer."""
    bufs = (buf0, buf1)
    for it in range(iters):
        _nb().nvbt_stencil(ctx, tools, bufs[it % 2], bufs[(it + 1) % 2], n, stream=stream)
    return bufs[iters % 2]


def replay_range(ctx, seed, first, n, hdr, addr, chunk=None):
    """Generate-then-replay events [first, first + n) in chunks that fit the given stream buffers."""
    cap = hdr.numel() // 16 if chunk is None else chunk
    done = 0
    while done < n:
        m = min(cap, n - done)
        _nb().nvbt_gen_events(ctx, seed, first + done, m, hdr, addr)
        _nb().nvbt_replay(ctx, hdr, addr, m)
        done += m


def merge_tensor(t, group=None):
    """Element-wise int64 SUM all-reduce of a packed accumulator tensor (any backend)."""
    import torch
    import torch.distributed as dist
    if t.dtype != torch.int64:
        raise TypeError("accumulators are int64")
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def merge(ctx, group=None):
    """a8: one int64 SUM all-reduce of the packed accumulator region (NCCL over NVLink on GPUs).
    Sums of disjoint event sets add (EM §4), so every rank then holds the whole job's result."""
    return merge_tensor(_nb().nvbt_accum_view(ctx), group)


class KernelSampler:
    """F1 kernel sampling (P:L274-282 (§6.2)): "we launch the instrumented version only once for each set
    of unique grid dimension values ... for the remaining ... times we run foo uninstrumented. We then use
    the information collected during the instrumented kernel execution to approximate the information not
    collected". The one instrumented launch of a key runs on a scratch context; its accumulator region is
    kept (device) and, at finish(), added to the target context once per launch of that key
    (nvbt_accum_axpy). When a kernel's control flow depends only on its grid dimensions the result is
    exact."""

    def __init__(self, ctx, scratch):
        self.ctx, self.scratch = ctx, scratch
        self.launches = {}
        self.snapshots = {}

    def launch(self, key, launch_fn, tools):
        """launch_fn(ctx_or_None, tools) enqueues one launch; key identifies its grid shape."""
        nb = _nb()
        self.launches[key] = self.launches.get(key, 0) + 1
        if key in self.snapshots:
            launch_fn(self.ctx, nb.TOOL_NONE)
            return False
        nb.nvbt_reset(self.scratch)
        launch_fn(self.scratch, tools)
        self.snapshots[key] = nb.nvbt_accum_view(self.scratch).clone()
        return True

    def finish(self):
        nb = _nb()
        for key, snap in self.snapshots.items():
            nb.nvbt_accum_axpy(self.ctx, snap, self.launches[key])
        return dict(self.launches)
