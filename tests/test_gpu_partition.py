"""Multi-GPU partitioning (SURVEY §8(e), row e) on the GPU.

* Single process: a context partitioned with nvbt_set_partition(ctx, r, w) runs rank r's share of every
  workload launch; the w ranks' accumulator regions must sum to the unpartitioned run's bit-exactly
  (partition invariance, I-6), and running every rank's share on the same buffers must reproduce the
  unpartitioned outputs (each output element has exactly one writer).
* Two processes on cuda:0 with the gloo backend (the driver's box has one GPU; gloo moves CUDA tensors
  through the host): the partitioned BFS with its per-level MAX exchanges and the partitioned stencil with
  its halo exchange, merged with the int64 SUM all-reduce (a8), against the CPU oracle."""
import os
import socket

import numpy as np
import pytest

from oracle import events as ev, programs
from oracle.models import bfs as m_bfs, stencil as m_st
from synth import uniform_f32, rmat_csr, bfs_source

from .gpu_util import read_all, assert_same

pytestmark = pytest.mark.gpu

COUNT_KEYS = ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t"]
MEM_KEYS = ["mem_n", "mem_S", "mem_L", "hS", "hL"]


def cuda(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def _sum_views(nb, ctxs):
    tot = nb.nvbt_accum_view(ctxs[0]).clone()
    for c in ctxs[1:]:
        tot += nb.nvbt_accum_view(c)
    return tot


def _check_partitioned(nb, workload, flags, n_warps, launch):
    """launch(ctx, out_index) runs one workload launch writing output set out_index (0: full, 1: shards)."""
    import torch
    full = nb.nvbt_init(workload, flags, n_warps=n_warps)
    launch(full, 0)
    for world in (2, 3, 7):
        ctxs = []
        for r in range(world):
            c = nb.nvbt_init(workload, flags, n_warps=n_warps)
            nb.nvbt_set_partition(c, r, world)
            launch(c, 1)
            ctxs.append(c)
        torch.cuda.synchronize()
        assert torch.equal(_sum_views(nb, ctxs), nb.nvbt_accum_view(full)), f"world {world}"
    return full


def test_partition_vectoradd_sgemm_stencil(nvbt):
    import torch
    nb = nvbt.nvbt
    flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP
    tools = nb.TOOL_COUNT | nb.TOOL_MEMDIV
    # C1 with a ragged tail; 2 CTAs only for N = 300 (world 3 and 7 leave ranks empty)
    for N in (65500, 300):
        a, b = cuda(uniform_f32(N, 1)), cuda(uniform_f32(N, 2))
        outs = [torch.empty_like(a), torch.full_like(a, -1.0)]
        nw = nb.nvbt_workload_warps(nb.W_VECTORADD, N)
        _check_partitioned(nb, nb.W_VECTORADD, flags, nw, lambda c, k: nb.nvbt_vectoradd(c, tools, a, b, outs[k], N))
        assert torch.equal(outs[0], outs[1])
    # C2 (2D CTA grid split along y)
    M, N, K = 96, 70, 33
    A, B = cuda(uniform_f32((M, K), 3, -1, 1)), cuda(uniform_f32((K, N), 4, -1, 1))
    outs = [torch.empty(M, N, device="cuda"), torch.full((M, N), -1.0, device="cuda")]
    nw = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
    _check_partitioned(nb, nb.W_SGEMM, flags, nw,
                       lambda c, k: nb.nvbt_sgemm(c, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV, A, B, outs[k], M, N, K))
    assert torch.equal(outs[0], outs[1])
    # C4 one iteration
    n = 100
    x0 = cuda(uniform_f32((n, n), 4))
    outs = [torch.empty_like(x0), torch.full_like(x0, -1.0)]
    nw = nb.nvbt_workload_warps(nb.W_STENCIL, n)
    _check_partitioned(nb, nb.W_STENCIL, flags, nw, lambda c, k: nb.nvbt_stencil(c, tools, x0, outs[k], n))
    assert torch.equal(outs[0], outs[1])


def test_partition_wfft(nvbt):
    import torch
    nb = nvbt.nvbt
    n_fft, ctas = 1000, 9
    g = torch.Generator(device="cuda").manual_seed(3)
    x = (torch.rand((n_fft, 32, 2), generator=g, device="cuda") * 2 - 1).view(torch.complex64).reshape(n_fft, 32)
    for w, v, t in ((nb.W_WFFT_EMU, nb.WFFT_PROXY, nb.TOOL_EMU | nb.TOOL_COUNT | nb.TOOL_MEMDIV),
                    (nb.W_WFFT_SW, nb.WFFT_SOFTWARE, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV)):
        outs = [torch.zeros_like(x), torch.zeros_like(x)]
        flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP
        _check_partitioned(nb, w, flags, 8 * ctas, lambda c, k: nb.nvbt_wfft32(c, t, v, x, outs[k], n_fft, ctas))
        assert torch.equal(outs[0].view(torch.int64), outs[1].view(torch.int64))


def test_partition_bfs_kernels_sum(nvbt):
    """Both BFS kernels partitioned on one process (no exchange needed when the ranks run one after the
    other on shared buffers): the summed accumulators equal the unpartitioned BFS."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    rowptr, col = rmat_csr(10, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    rp, cl = cuda(rowptr), cuda(col)
    flags = nb.COUNT | nb.BB | nb.MEMDIV
    tools = nb.TOOL_COUNT | nb.TOOL_MEMDIV
    full = nb.nvbt_init(nb.W_BFS, flags)
    cost_full, lv = dr.run_bfs(full, tools, rp, cl, src)
    world = 3
    ctxs = [nb.nvbt_init(nb.W_BFS, flags) for _ in range(world)]
    for r, c in enumerate(ctxs):
        nb.nvbt_set_partition(c, r, world)
    b = dr.bfs_buffers(n, "cuda")
    b["mask"][src] = 1; b["visited"][src] = 1; b["cost"][src] = 0
    for level in range(lv):
        b["over"].zero_(); b["updating"].zero_()
        for c in ctxs:
            nb.nvbt_bfs_expand(c, tools, rp, cl, n, b["mask"], b["visited"], b["updating"])
        for c in ctxs:
            nb.nvbt_bfs_update(c, tools, n, b["mask"], b["visited"], b["updating"], b["cost"], b["over"], level)
    torch.cuda.synchronize()
    assert torch.equal(b["cost"], cost_full)
    assert torch.equal(_sum_views(nb, ctxs), nb.nvbt_accum_view(full))


def test_partition_errors(nvbt):
    nb = nvbt.nvbt
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT)
    for r, w in ((0, 0), (2, 2), (5, 3)):
        with pytest.raises(nb.NvbtError):
            nb.nvbt_set_partition(ctx, r, w)


# ---------------------------------------------------------------- two processes, gloo, one GPU
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_micro_villasnk19_b200 as pkg
        nb, dr = pkg.nvbt, pkg.drivers
        out = {}
        # C3: partitioned BFS with per-level exchanges
        rowptr, col = rmat_csr(11, 16, seed=3)
        n = len(rowptr) - 1
        src = bfs_source(rowptr)
        rp, cl = cuda(rowptr), cuda(col)
        ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB | nb.MEMDIV)
        nb.nvbt_set_partition(ctx, rank, world)
        bufs = dr.bfs_buffers(n, "cuda")
        cost, levels = dr.run_bfs_dist(ctx, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV, rp, cl, src, bufs)
        dr.merge(ctx)
        out["bfs"] = (read_all(nb, ctx), cost.cpu().numpy(), levels,
                      [bufs[k].data_ptr() for k in ("mask", "visited", "updating", "cost", "over")],
                      rp.data_ptr(), cl.data_ptr())
        # C4: partitioned stencil with halo exchange, trace digests merged
        sn, iters = 96, 3
        sctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.MEMDIV | nb.TRACE)
        nb.nvbt_set_partition(sctx, rank, world)
        ring = torch.empty(nb.nvbt_channel_bytes(1 << 14), dtype=torch.uint8, pin_memory=True)
        ch = nb.nvbt_channel_open(sctx, ring)
        x0 = cuda(uniform_f32((sn, sn), 4))
        b0, b1 = x0.clone(), torch.zeros_like(x0)
        fin = dr.run_stencil_dist(sctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV | nb.TOOL_TRACE, b0, b1, sn, iters, rank, world)
        d = nb.nvbt_channel_drain_digest(ch, timeout_us=60_000_000)
        dr.merge(sctx)
        # records carry this process's buffer addresses: the parent checks each rank's digest on its own
        out["stencil"] = (read_all(nb, sctx), fin.cpu().numpy(), x0.cpu().numpy(), b0.data_ptr(), b1.data_ptr())
        q.put((rank, (d.n_rec, d.d1, d.d2, b0.data_ptr(), b1.data_ptr()), out if rank == 0 else None))
    finally:
        dist.destroy_process_group()


def test_two_rank_bfs_and_stencil_exchanges(nvbt):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    msgs = dict((r, (dg, o)) for r, dg, o in (q.get(timeout=600) for _ in range(2)))
    out = msgs[0][1]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    # C3 against the oracle's single-GPU BFS model (same buffer addresses as rank 0's)
    g, cost, levels, ptrs, rpp, clp = out["bfs"]
    rowptr, col = rmat_csr(11, 16, seed=3)
    src = bfs_source(rowptr)
    acc = ev.Accumulator(programs.bfs())
    ocost, olevels, _ = m_bfs.run(acc, rowptr, col, src, m_bfs.Ptrs(*ptrs, rpp, clp))
    assert levels == olevels and (cost == ocost).all()
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS, "2-rank BFS")
    # C4: merged counts, divergence and trace digests == oracle; gathered grid == Jacobi reference
    g, fin, x0, p0, p1 = out["stencil"]
    acc = ev.Accumulator(programs.stencil())
    m_st.run_iterations(acc, 96, p0, p1, 3)
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS, "2-rank stencil")
    assert np.array_equal(fin, m_st.jacobi_reference(x0, 3))
    gx, gy = 96 // 32, 96 // 8
    for r in (0, 1):                                   # rank r's records: its warps, its buffers
        n_rec, d1, d2, q0, q1 = msgs[r][0]
        y0, y1 = gy * r // 2, gy * (r + 1) // 2
        racc = ev.Accumulator(programs.stencil(), trace=True)
        m_st.run_iterations(racc, 96, q0, q1, 3, warps=np.arange(8 * gx * y0, 8 * gx * y1))
        assert (n_rec, d1, d2) == (racc.digest.n, racc.digest.d1, racc.digest.d2), f"rank {r} trace"
