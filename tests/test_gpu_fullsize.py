"""GPU parity at BASELINE.json's full sizes, element by element against the multithreaded C oracle
(oracle/coracle.py; pinned in tests/test_oracle_c.py), in the launch configurations bench.py times.

  C2  naive SGEMM 1024^3, COUNT|MEMDIV|PER_WARP and the bench's BBCOUNT|MEMDIV
  C3  BFS on the R-MAT scale-20 graph, COUNT|MEMDIV|PER_WARP and BBCOUNT
  C4  stencil 8192^2 x 100 with COUNT|MEMDIV|TRACE in ONE run through the pinned-host channel: counts,
      histograms, per-pc divergence and the trace multiset digest (N_rec, D1, D2), plus SURVEY I-3's
      ΣS = 5,450,035,600 and ΣL = 1,675,776,400; then the same trace through both compact transports
  C5  all 10^10 generated events through the staged replay in 2^27-event chunks (and the single-pass
      kernel on the same chunks)

Every accumulator the C ABI reports is compared (counts, H_t/H_w, Ent/Ins per block, per-pc n/ΣS/ΣL,
hS/hL, per-warp arrays where enabled). The oracle runs on all host cores, concurrently with the GPU
where the GPU path does not need the host (C5)."""
import threading

import numpy as np
import pytest

from oracle import coracle as co, programs, gen
from synth import uniform_f32, rmat_csr, bfs_source

from .gpu_util import read_all, assert_same, gpu_invariants

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

COUNT_KEYS = ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t"]
MEM_KEYS = ["mem_n", "mem_S", "mem_L", "hS", "hL"]


def cuda(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


class Background:
    """Runs an oracle call on a host thread (ctypes releases the GIL) while the GPU works."""

    def __init__(self, fn, *a, **kw):
        self.res, self.err = None, None

        def run():
            try:
                self.res = fn(*a, **kw)
            except BaseException as e:  # noqa: BLE001 - re-raised in get()
                self.err = e
        self.t = threading.Thread(target=run)
        self.t.start()

    def get(self):
        self.t.join()
        if self.err:
            raise self.err
        return self.res


def test_c2_sgemm_full_size(nvbt):
    import torch
    nb = nvbt.nvbt
    M = N = K = 1024
    nw = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
    A = cuda(uniform_f32((M, K), 3, -1, 1))
    B = cuda(uniform_f32((K, N), 4, -1, 1))
    Cm = torch.empty(M, N, device="cuda")
    ref = Background(co.sgemm, programs.sgemm(), M, N, K, A.data_ptr(), B.data_ptr(), Cm.data_ptr(), per_warp=True)
    got = {}
    for name, tools in (("count", nb.TOOL_COUNT | nb.TOOL_MEMDIV), ("bench", nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV)):
        ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
        nb.nvbt_sgemm(ctx, tools, A, B, Cm, M, N, K)
        got[name] = read_all(nb, ctx, per_warp=True)
    r = ref.get()
    for name, g in got.items():
        assert_same(g, r, COUNT_KEYS + MEM_KEYS + ["PW_T", "PW_W"], f"C2 1024^3 {name}")
    assert int(r["mem_S"].sum()) == int(r["mem_L"].sum()) == 1_108_344_832
    gpu_invariants(got["count"])


def test_c3_bfs_full_size(nvbt):
    nb, dr = nvbt.nvbt, nvbt.drivers
    rowptr, col = rmat_csr(20, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    nw = nb.nvbt_workload_warps(nb.W_BFS, n)
    rp, cl = cuda(rowptr), cuda(col)
    for name, tools in (("count", nb.TOOL_COUNT | nb.TOOL_MEMDIV), ("bb", nb.TOOL_BBCOUNT)):
        ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
        bufs = dr.bfs_buffers(n, "cuda")
        cost, levels = dr.run_bfs(ctx, tools, rp, cl, src, bufs)
        g = read_all(nb, ctx, per_warp=True)
        ptrs = [bufs[k].data_ptr() for k in ("mask", "visited", "updating", "cost", "over")] + \
               [rp.data_ptr(), cl.data_ptr()]
        r, ocost, olevels = co.bfs(programs.bfs(), rowptr, col, src, ptrs, per_warp=True)
        assert levels == olevels and np.array_equal(cost.cpu().numpy(), ocost)
        if name == "count":   # the BFS itself against scipy's unweighted shortest paths (I-4)
            from scipy.sparse import csr_matrix
            from scipy.sparse.csgraph import shortest_path
            Ag = csr_matrix((np.ones(len(col), dtype=np.int8), col, rowptr), shape=(n, n))
            dist = shortest_path(Ag, unweighted=True, indices=src)
            assert np.array_equal(ocost.astype(np.int64), np.where(np.isinf(dist), -1, dist).astype(np.int64))
        keys = COUNT_KEYS + ["PW_T", "PW_W"] + (MEM_KEYS if name == "count" else [])
        assert_same(g, r, keys, f"C3 scale 20 {name}")
        gpu_invariants(g)


def test_c4_stencil_trace_full_size(nvbt):
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n, iters = 8192, 100
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.TRACE)
    x0 = cuda(uniform_f32((n, n), 4))
    b0, b1 = x0.clone(), torch.empty_like(x0)
    ring = torch.empty(nb.nvbt_channel_bytes(1 << 22), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring)
    dr.run_stencil(ctx, nb.TOOL_TRACE | nb.TOOL_COUNT | nb.TOOL_MEMDIV, b0, b1, n, iters)
    d = nb.nvbt_channel_drain_digest(ch, timeout_us=900_000_000)
    torch.cuda.synchronize()
    assert nb.nvbt_channel_dropped(ch) == 0
    g = read_all(nb, ctx)
    r = co.stencil(programs.stencil(), n, b0.data_ptr(), b1.data_ptr(), iters, trace=True)
    assert_same(g, r, COUNT_KEYS + MEM_KEYS, "C4 8192^2 x 100")
    assert (d.n_rec, d.d1, d.d2) == tuple(int(x) for x in r["trace"]), "C4 trace multiset digest"
    assert d.n_rec == 1_258_086_400
    assert int(g["mem_S"].sum()) == 5_450_035_600 and int(g["mem_L"].sum()) == 1_675_776_400
    gpu_invariants(g)
    nb.nvbt_channel_close(ch)
    del ring
    # the same 100 launches (launch ids restart at reset, same buffers: the same record multiset) through
    # the two compact transports (F3, EM §5.1 / §5.2), decoded on the host: identical digests
    for compact in (True, 128):
        nb.nvbt_reset(ctx)
        ring = torch.empty(nb.nvbt_channel_bytes(1 << 22, compact=compact), dtype=torch.uint8, pin_memory=True)
        ch = nb.nvbt_channel_open(ctx, ring, compact=compact)
        dr.run_stencil(ctx, nb.TOOL_TRACE, b0, b1, n, iters)
        dc = nb.nvbt_channel_drain_digest(ch, timeout_us=900_000_000)
        torch.cuda.synchronize()
        assert nb.nvbt_channel_dropped(ch) == 0
        assert (dc.n_rec, dc.d1, dc.d2) == tuple(int(x) for x in r["trace"]), f"C4 compact={compact} digest"
        nb.nvbt_channel_close(ch)
        del ring


def test_c5_replay_full_size(nvbt):
    import torch
    nb = nvbt.nvbt
    n, chunk = 10**10, 1 << 27
    ref = Background(co.replay, programs.replay(), gen.SEED, 0, n)
    flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV
    hdr = torch.empty(chunk * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty(chunk * 256, dtype=torch.uint8, device="cuda")
    ctx = nb.nvbt_init(nb.W_REPLAY, flags)
    single = nb.nvbt_init(nb.W_REPLAY, flags)          # the single-pass kernel on the same stream
    scratch = torch.empty(nb.nvbt_replay_scratch_size(ctx, chunk), dtype=torch.uint8, device="cuda")
    done = 0
    while done < n:
        m = min(chunk, n - done)
        nb.nvbt_gen_events(ctx, gen.SEED, done, m, hdr, addr)
        nb.nvbt_replay_staged(ctx, hdr, addr, m, scratch)
        nb.nvbt_replay(single, hdr, addr, m)
        done += m
    g = read_all(nb, ctx)
    assert nb.nvbt_replay_errors(ctx) == 0 and nb.nvbt_replay_errors(single) == 0
    assert_same(read_all(nb, single), g, COUNT_KEYS + MEM_KEYS, "C5 single-pass vs staged")
    del hdr, addr, scratch
    torch.cuda.empty_cache()
    r = ref.get()
    assert_same(g, r, COUNT_KEYS + MEM_KEYS, "C5 10^10 events")
    assert int(g["counts"][2]) == n
    gpu_invariants(g)
