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


# ------------------------------------------------------------------ multi-GPU partitioned workloads
def cta_rows(gy: int, rank: int, world: int):
    """CTA rows [y0, y1) of a gy-row CTA grid that rank runs (the rule nvbt_set_partition documents)."""
    return gy * rank // world, gy * (rank + 1) // world


def run_bfs_dist(ctx, tools, rowptr, col, src, bufs=None, group=None, max_levels=1 << 20):
    """C3 over `world` ranks: ctx is partitioned (nvbt_set_partition), so each rank runs
    both BFS kernels on its own vertex range; the graph is replicated. Per level: every rank clears
    `updating`, runs kernel 1 (it marks any neighbour, owned or not), MAX-all-reduces `updating`, runs
    kernel 2 on its own vertices, then MAX-all-reduces `visited` and `over`. At the end `cost` (−1 outside
    a rank's own vertices) is MAX-all-reduced. Every instrumented warp runs on exactly one rank, so the
    ranks' accumulators sum to the single-GPU result (merge()). Returns (cost, levels)."""
    import torch
    import torch.distributed as dist
    nb = _nb()
    n = rowptr.numel() - 1
    b = bfs_buffers(n, rowptr.device) if bufs is None else bufs
    b["mask"].zero_(); b["visited"].zero_(); b["updating"].zero_(); b["cost"].fill_(-1)
    b["mask"][src] = 1
    b["visited"][src] = 1
    b["cost"][src] = 0
    level = 0
    while level < max_levels:
        b["over"].zero_()
        b["updating"].zero_()
        nb.nvbt_bfs_expand(ctx, tools, rowptr, col, n, b["mask"], b["visited"], b["updating"])
        _sync(ctx)
        dist.all_reduce(b["updating"], op=dist.ReduceOp.MAX, group=group)
        nb.nvbt_bfs_update(ctx, tools, n, b["mask"], b["visited"], b["updating"], b["cost"], b["over"], level)
        _sync(ctx)
        dist.all_reduce(b["visited"], op=dist.ReduceOp.MAX, group=group)
        dist.all_reduce(b["over"], op=dist.ReduceOp.MAX, group=group)
        level += 1
        if int(b["over"].item()) == 0:
            break
    dist.all_reduce(b["cost"], op=dist.ReduceOp.MAX, group=group)
    return b["cost"], level


def stencil_rows(n: int, rank: int, world: int):
    """Grid rows [r0, r1) a rank computes in the partitioned stencil (CTA rows of 8 grid rows)."""
    y0, y1 = cta_rows((n + 7) // 8, rank, world)
    return min(8 * y0, n), min(8 * y1, n)


def slab_neighbours(n: int, rank: int, world: int):
    """Nearest ranks above and below `rank` whose row slabs are non-empty (None at the grid's edges). A
    rank with an empty slab sits between them with r0 == r1, so the neighbour above ends exactly at my
    first row and the one below starts right after my last row."""
    up = next((q for q in range(rank - 1, -1, -1) if stencil_rows(n, q, world)[1] > stencil_rows(n, q, world)[0]), None)
    down = next((q for q in range(rank + 1, world) if stencil_rows(n, q, world)[1] > stencil_rows(n, q, world)[0]), None)
    return up, down


def _backend(group):
    import torch.distributed as dist
    return dist.get_backend(group)


def _exchange_halo(buf, n, rank, world, group):
    """1-row halos with the two slab neighbours ("1-row halos (32 KiB) via P2P send/recv"):
    send my first row up and my last row down, receive the row above my slab and the row below it.
    NCCL: one batched isend/irecv group, stream-ordered after the iteration's kernel (no host sync, so
    the trace drain keeps running); other backends (gloo, CPU tests) stage the rows through the host."""
    import torch
    import torch.distributed as dist
    r0, r1 = stencil_rows(n, rank, world)
    if r1 == r0:                     # an empty slab computes nothing and needs no halo
        return
    up, down = slab_neighbours(n, rank, world)
    g = buf.view(torch.int32)
    nccl = _backend(group) == "nccl"
    pairs = []                        # (peer, row to send, row to receive into)
    if up is not None:
        pairs.append((up, r0, r0 - 1))
    if down is not None:
        pairs.append((down, r1 - 1, r1))
    if not pairs:
        return
    gr = (lambda q: q) if group is None else (lambda q: dist.get_global_rank(group, q))
    if nccl:
        ops = []
        for peer, srow, rrow in pairs:
            ops.append(dist.P2POp(dist.isend, g[srow], gr(peer), group))
            ops.append(dist.P2POp(dist.irecv, g[rrow], gr(peer), group))
        for w in dist.batch_isend_irecv(ops):
            w.wait()
        return
    host = [(peer, g[srow].cpu(), torch.empty(n, dtype=torch.int32), rrow) for peer, srow, rrow in pairs]
    ops = []
    for peer, sbuf, rbuf, _ in host:
        ops.append(dist.P2POp(dist.isend, sbuf, gr(peer), group))
        ops.append(dist.P2POp(dist.irecv, rbuf, gr(peer), group))
    for w in dist.batch_isend_irecv(ops):
        w.wait()
    for _, _, rbuf, rrow in host:
        g[rrow].copy_(rbuf)


def run_stencil_dist(ctx, tools, buf0, buf1, n, iters, rank, world, group=None, gather=True):
    """C4 over `world` ranks: ctx is partitioned, so each rank runs the CTA rows of its own
    row slab; after every iteration the 1-row halos go to and come from the slab neighbours
    (_exchange_halo). Under NCCL nothing here waits on the host, so a caller can enqueue all iterations
    and drain the trace channel while they run. With `gather`, the full final grid is assembled on every
    rank at the end (one int32 SUM all-reduce, rows outside a rank's slab zeroed first). Trace records stay
    on each rank's own channel; their digests add. Returns the final buffer."""
    import torch
    import torch.distributed as dist
    bufs = (buf0, buf1)
    stream = getattr(ctx, "stream", None)
    with torch.cuda.stream(stream) if stream is not None else _null():
        for it in range(iters):
            _nb().nvbt_stencil(ctx, tools, bufs[it % 2], bufs[(it + 1) % 2], n)
            _exchange_halo(bufs[(it + 1) % 2], n, rank, world, group)
        out = bufs[iters % 2]
        if gather:
            r0, r1 = stencil_rows(n, rank, world)
            g = out.view(torch.int32)
            g[:r0] = 0
            g[r1:] = 0
            dist.all_reduce(g, op=dist.ReduceOp.SUM, group=group)
    return out


class _null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


def replay_range(ctx, seed, first, n, hdr, addr, chunk=None, scratch=None):
    """Generate-then-replay events [first, first + n) in chunks that fit the given stream buffers; with a
    scratch tensor the staged two-pass replay (nvbt_replay_staged) runs instead of the single pass."""
    cap = hdr.numel() // 16 if chunk is None else chunk
    done = 0
    while done < n:
        m = min(cap, n - done)
        _nb().nvbt_gen_events(ctx, seed, first + done, m, hdr, addr)
        if scratch is None:
            _nb().nvbt_replay(ctx, hdr, addr, m)
        else:
            _nb().nvbt_replay_staged(ctx, hdr, addr, m, scratch)
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


# --------------------------------------------------------------------------- host placement of a rank
# A traced rank moves its records over its GPU's own PCIe link into a pinned ring that its drain threads
# scan (C4). On a multi-socket box each GPU hangs off one NUMA node: the ring pages and the drain threads
# belong on that node, and the ranks sharing a node split its cores instead of all spinning on all of them.

def parse_cpulist(text: str):
    """'0-3,8,10-11' -> [0, 1, 2, 3, 8, 10, 11] (the sysfs cpulist format)."""
    cpus = []
    for part in text.strip().split(","):
        if not part:
            continue
        if "-" in part:
            lo, hi = part.split("-")
            cpus.extend(range(int(lo), int(hi) + 1))
        else:
            cpus.append(int(part))
    return cpus


def rank_cpu_slice(gpu_cpus, device: int, allowed=None):
    """CPUs for the rank driving GPU `device`, given gpu_cpus[g] = the CPUs local to visible GPU g: the GPUs
    with the same local CPU set share it in contiguous equal slices (in GPU order), restricted to `allowed`
    (the process's affinity). Falls back to the whole local set (or `allowed`) when a slice would be empty."""
    mine = [c for c in gpu_cpus[device] if allowed is None or c in allowed]
    peers = [g for g, cs in enumerate(gpu_cpus) if sorted(cs) == sorted(gpu_cpus[device])]
    k, i = len(peers), peers.index(device)
    lo, hi = len(mine) * i // k, len(mine) * (i + 1) // k
    if hi > lo:
        return mine[lo:hi]
    return mine or (sorted(allowed) if allowed else [])


def gpu_local_cpus(sysfs="/sys/bus/pci/devices"):
    """Per visible CUDA device, the CPUs of its PCIe device's NUMA node (sysfs local_cpulist); None if the
    topology cannot be read."""
    import torch
    out = []
    for g in range(torch.cuda.device_count()):
        p = torch.cuda.get_device_properties(g)
        dev = f"{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
        try:
            with open(f"{sysfs}/{dev}/local_cpulist") as f:
                out.append(parse_cpulist(f.read()))
        except OSError:
            return None
    return out


def bind_rank_to_gpu_numa(device: int):
    """Pins this process to its slice of GPU `device`'s NUMA-local CPUs (call before the pinned ring is
    allocated and before the first drain creates the drain worker pool, which sizes itself to the affinity).
    Returns the CPU list, or None when the topology is unknown (nothing changed)."""
    import os
    local = gpu_local_cpus()
    if not local:
        return None
    cpus = rank_cpu_slice(local, device, set(os.sched_getaffinity(0)))
    if not cpus:
        return None
    os.sched_setaffinity(0, cpus)
    return cpus
