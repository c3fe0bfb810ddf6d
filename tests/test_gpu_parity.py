"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

Every input is seeded; addresses in events are the real device addresses, which the oracle models
receive as inputs. Sizes span several CTAs and ragged tails; full-size cases check closed forms, the
oracle on sampled warps and invariants."""
import numpy as np
import pytest

from oracle import events as ev, programs, gen, trace
from oracle.models import vectoradd as m_va, sgemm as m_sg, stencil as m_st, bfs as m_bfs
from synth import uniform_f32, rmat_csr, bfs_source

from .gpu_util import read_all, assert_same, gpu_invariants

pytestmark = pytest.mark.gpu

COUNT_KEYS = ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t"]
MEM_KEYS = ["mem_n", "mem_S", "mem_L", "hS", "hL"]


def cuda(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


# ---------------------------------------------------------------- C1 vectorAdd
@pytest.mark.parametrize("N", [65536, 65500, 1000, 31, 257])
@pytest.mark.parametrize("count_tool", ["COUNT", "BBCOUNT"])
def test_vectoradd_parity(nvbt, N, count_tool):
    import torch
    nb = nvbt.nvbt
    tools = getattr(nb, "TOOL_" + count_tool) | nb.TOOL_MEMDIV
    nw = nb.nvbt_workload_warps(nb.W_VECTORADD, N)
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
    a, b = cuda(uniform_f32(N, 1)), cuda(uniform_f32(N, 2))
    c = torch.empty_like(a)
    nb.nvbt_vectoradd(ctx, tools, a, b, c, N)
    g = read_all(nb, ctx, per_warp=True)
    acc = ev.Accumulator(programs.vectoradd(), n_warps=nw)
    m_va.run(acc, N, a.data_ptr(), b.data_ptr(), c.data_ptr())
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS + ["PW_T", "PW_W"], f"vectorAdd N={N} {count_tool}")
    assert torch.equal(c, a + b)
    gpu_invariants(g)


def test_vectoradd_plain_and_cumulative(nvbt):
    """Uninstrumented launches count nothing; instrumented results accumulate until reset."""
    import torch
    nb = nvbt.nvbt
    N = 4096
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT)
    a, b = cuda(uniform_f32(N, 1)), cuda(uniform_f32(N, 2))
    c = torch.empty_like(a)
    nb.nvbt_vectoradd(ctx, nb.TOOL_NONE, a, b, c, N)
    assert (nb.nvbt_count(ctx) == 0).all()
    nb.nvbt_vectoradd(ctx, nb.TOOL_COUNT, a, b, c, N)
    one = nb.nvbt_count(ctx).copy()
    nb.nvbt_vectoradd(ctx, nb.TOOL_COUNT, a, b, c, N)
    assert (nb.nvbt_count(ctx) == 2 * one).all()
    nb.nvbt_reset(ctx)
    assert (nb.nvbt_count(ctx) == 0).all()
    with pytest.raises(nb.NvbtError):            # MEMDIV not enabled at init
        nb.nvbt_vectoradd(ctx, nb.TOOL_MEMDIV, a, b, c, N)
    with pytest.raises(nb.NvbtError):            # wrong program for this context
        nb.nvbt_sgemm(ctx, nb.TOOL_COUNT, a, b, c, 32, 8, 1)


# ---------------------------------------------------------------- C2 SGEMM
@pytest.mark.parametrize("M,N,K", [(64, 32, 48), (100, 20, 5), (33, 9, 1), (96, 64, 130)])
@pytest.mark.parametrize("tools", ["COUNT|MEMDIV", "BBCOUNT|MEMDIV", "MEMDIV"])
def test_sgemm_parity(nvbt, M, N, K, tools):
    import torch
    nb = nvbt.nvbt
    t = 0
    for x in tools.split("|"):
        t |= getattr(nb, "TOOL_" + x)
    nw = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
    ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
    A = cuda(uniform_f32((M, K), 3, -1, 1))
    B = cuda(uniform_f32((K, N), 4, -1, 1))
    Cm = torch.empty(M, N, device="cuda")
    nb.nvbt_sgemm(ctx, t, A, B, Cm, M, N, K)
    g = read_all(nb, ctx, per_warp=True)
    acc = ev.Accumulator(programs.sgemm(), n_warps=nw)
    m_sg.run(acc, M, N, K, A.data_ptr(), B.data_ptr(), Cm.data_ptr())
    ref = acc.result()
    keys = MEM_KEYS + (COUNT_KEYS + ["PW_T", "PW_W"] if "COUNT" in tools else [])
    assert_same(g, ref, keys, f"SGEMM {M}x{N}x{K} {tools}")
    torch.testing.assert_close(Cm, A @ B, rtol=1e-4, atol=1e-4)


# ---------------------------------------------------------------- C3 BFS
@pytest.mark.parametrize("scale,tools", [(12, "BBCOUNT"), (12, "COUNT|MEMDIV"), (10, "BBCOUNT|MEMDIV")])
def test_bfs_parity(nvbt, scale, tools):
    nb, dr = nvbt.nvbt, nvbt.drivers
    t = 0
    for x in tools.split("|"):
        t |= getattr(nb, "TOOL_" + x)
    rowptr, col = rmat_csr(scale, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    nw = nb.nvbt_workload_warps(nb.W_BFS, n)
    ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw)
    rp, cl = cuda(rowptr), cuda(col)
    bufs = dr.bfs_buffers(n, "cuda")
    cost, levels = dr.run_bfs(ctx, t, rp, cl, src, bufs)
    g = read_all(nb, ctx, per_warp=True)
    acc = ev.Accumulator(programs.bfs(), n_warps=nw)
    ptr = m_bfs.Ptrs(bufs["mask"].data_ptr(), bufs["visited"].data_ptr(), bufs["updating"].data_ptr(),
                     bufs["cost"].data_ptr(), bufs["over"].data_ptr(), rp.data_ptr(), cl.data_ptr())
    ocost, olevels, _ = m_bfs.run(acc, rowptr, col, src, ptr)
    assert levels == olevels
    assert (cost.cpu().numpy() == ocost).all()
    ref = acc.result()
    keys = (COUNT_KEYS + ["PW_T", "PW_W"]) + (MEM_KEYS if "MEMDIV" in tools else [])
    assert_same(g, ref, keys, f"BFS scale {scale} {tools}")


# ---------------------------------------------------------------- C4 stencil + trace channel
def _stencil_case(nvbt, n, iters, ring_records, tools_names=("TRACE", "MEMDIV", "COUNT"), compact=False):
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    t = 0
    for x in tools_names:
        t |= getattr(nb, "TOOL_" + x)
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.MEMDIV | nb.TRACE)
    x0 = cuda(uniform_f32((n, n), 4))
    buf0, buf1 = x0.clone(), torch.zeros_like(x0)
    ring = torch.empty(nb.nvbt_channel_bytes(ring_records, compact=compact), dtype=torch.uint8, pin_memory=True)
    ring.view(torch.int32).fill_(1)            # stale "lap 1" tags everywhere: open must clear them
    ch = nb.nvbt_channel_open(ctx, ring, compact=compact)
    dr.run_stencil(ctx, t, buf0, buf1, n, iters)
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    m_st.run_iterations(acc, n, buf0.data_ptr(), buf1.data_ptr(), iters)
    exp = acc.record_array()
    dst = np.zeros((len(exp) + 65536, 288), dtype=np.uint8)
    got_n = nb.nvbt_channel_drain_copy(ch, dst, timeout_us=60_000_000)
    assert nb.nvbt_channel_dropped(ch) == 0
    got = dst[:got_n]
    ids, cnt = np.unique(got.view("<u4")[:, 0], return_counts=True)
    assert got_n == len(exp), f"launch ids {ids} x {cnt}"

    assert (trace.sort_records(got) == trace.sort_records(exp)).all()
    out = buf0 if iters % 2 == 0 else buf1
    ref_grid = m_st.jacobi_reference(x0.cpu().numpy(), iters)
    assert np.array_equal(out.cpu().numpy(), ref_grid)
    return ctx, acc, got


@pytest.mark.parametrize("n,iters", [(96, 3), (100, 2), (64, 1)])
def test_stencil_trace_parity(nvbt, n, iters):
    nb = nvbt.nvbt
    ctx, acc, got = _stencil_case(nvbt, n, iters, ring_records=1 << 16)
    g = read_all(nb, ctx)
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS, f"stencil n={n}")
    assert nb.nvbt_digest_records(got) == (acc.digest.n, acc.digest.d1, acc.digest.d2)


def test_channel_tiny_ring_backpressure(nvbt):
    """A 5-slot ring forces wrap-around and producer backpressure; nothing lost or duplicated."""
    _stencil_case(nvbt, 64, 2, ring_records=5, tools_names=("TRACE",))


@pytest.mark.parametrize("force_wide,ring", [("0", 1 << 16), ("0", 5), ("1", 1 << 16), ("1", 7), ("1", 6)])
def test_channel_compact_transport(nvbt, monkeypatch, force_wide, ring):
    """F3 compact 176 B slots (EM §5.1): decoded records equal the oracle's; the forced wide form (two
    slots per record) with odd and even tiny rings exercises pairs straddling the ring end."""
    monkeypatch.setenv("NVBT_COMPACT_FORCE_WIDE", force_wide)
    _stencil_case(nvbt, 64, 2, ring_records=ring, tools_names=("TRACE", "MEMDIV"), compact=True)


@pytest.mark.parametrize("force_long,ring", [("0", 1 << 16), ("0", 5), ("1", 1 << 16), ("1", 7), ("1", 4), ("1", 3)])
def test_channel_compact128_transport(nvbt, monkeypatch, force_long, ring):
    """EM §5.2 128 B slots: decoded records equal the oracle's; the forced three-slot form on 3/4/7-slot
    rings exercises records straddling the ring end (the drain stashes their first slots)."""
    monkeypatch.setenv("NVBT_COMPACT_FORCE_WIDE", force_long)
    _stencil_case(nvbt, 64, 2, ring_records=ring, tools_names=("TRACE", "MEMDIV"), compact=128)


def test_channel_compact128_bfs(nvbt):
    """BFS records (gathers across MBs) need the three-slot form of EM §5.2; mixed with one-slot records on
    a small ring, every record arrives intact (multiset == the oracle's)."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    rowptr, col = rmat_csr(10, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    ctx = nb.nvbt_init(nb.W_BFS, nb.TRACE)
    rp, cl = cuda(rowptr), cuda(col)
    bufs = dr.bfs_buffers(n, "cuda")
    ring = torch.empty(nb.nvbt_channel_bytes(1 << 10, compact=128), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring, compact=128)
    acc = ev.Accumulator(programs.bfs(), trace=True, keep_records=True)
    ptr = m_bfs.Ptrs(bufs["mask"].data_ptr(), bufs["visited"].data_ptr(), bufs["updating"].data_ptr(),
                     bufs["cost"].data_ptr(), bufs["over"].data_ptr(), rp.data_ptr(), cl.data_ptr())
    m_bfs.run(acc, rowptr, col, src, ptr)
    exp = acc.record_array()
    dst = np.zeros((len(exp) + 1024, 288), dtype=np.uint8)
    got_n = 0
    import threading
    done, out = threading.Event(), []

    import os
    import time
    log = []
    t0 = time.perf_counter()

    def drain():   # the ring (1024 slots) is far smaller than the trace: drain while the BFS runs
        log.append(("start", time.perf_counter() - t0, sorted(os.sched_getaffinity(0))[:4]))
        try:
            while True:
                fin = done.is_set()
                a = time.perf_counter() - t0
                out.append(nb.nvbt_channel_drain_copy(ch, dst[sum(out):], timeout_us=60_000_000))
                log.append((round(a, 4), round(time.perf_counter() - t0, 4), out[-1]))
                if fin:
                    return
        except Exception as e:  # noqa: BLE001 - reported with the log below
            log.append(("error", time.perf_counter() - t0, str(e)))
    th = threading.Thread(target=drain)
    th.start()
    dr.run_bfs(ctx, nb.TOOL_TRACE, rp, cl, src, bufs)
    log.append(("bfs done", time.perf_counter() - t0))
    done.set()
    th.join()
    got_n = sum(out)
    assert nb.nvbt_channel_dropped(ch) == 0 and got_n == len(exp), (got_n, len(exp), log[:20], log[-5:], threading.enumerate())
    assert (trace.sort_records(dst[:got_n]) == trace.sort_records(exp)).all()


def test_channel_drop_is_reported(nvbt, monkeypatch):
    """A host ring nobody drains while the kernel runs: the producers wait (here 2 s, NVBT_PRODUCER_WAIT_MS)
    for room, then give up; the
    records they drop are counted (nvbt_channel_dropped) and the drain fails loudly (NVBT_ETIMEDOUT) after
    delivering what was committed, instead of hanging or passing silently (include/nvbt.h: the channel
    must then be reopened)."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n = 64
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.TRACE)
    x0 = cuda(uniform_f32((n, n), 4))
    b0, b1 = x0.clone(), torch.zeros_like(x0)
    ring = torch.empty(nb.nvbt_channel_bytes(8), dtype=torch.uint8, pin_memory=True)
    monkeypatch.setenv("NVBT_PRODUCER_WAIT_MS", "2000")
    ch = nb.nvbt_channel_open(ctx, ring)
    dr.run_stencil(ctx, nb.TOOL_TRACE, b0, b1, n, 1)
    torch.cuda.synchronize()                     # no consumer ran: the ring filled up
    dropped = nb.nvbt_channel_dropped(ch)
    assert dropped > 0
    dst = np.zeros((1024, 288), dtype=np.uint8)
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_channel_drain_copy(ch, dst, timeout_us=30_000_000)
    assert e.value.code == nb.ETIMEDOUT and "dropped" in str(e.value)
    nb.nvbt_channel_close(ch)
    ch = nb.nvbt_channel_open(ctx, ring)          # a reopened channel works again
    nb.nvbt_reset(ctx)
    dr.run_stencil(ctx, nb.TOOL_TRACE, b0, b1, n, 1)
    G = n // 32
    got = nb.nvbt_channel_drain_copy(ch, dst, timeout_us=30_000_000)   # drains while the kernel runs
    assert got == 4 * G + 6 * G * (n - 2) and nb.nvbt_channel_dropped(ch) == 0


def test_channel_digest_drain(nvbt):
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n, iters = 128, 2
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.TRACE)
    x0 = cuda(uniform_f32((n, n), 4))
    buf0, buf1 = x0.clone(), torch.zeros_like(x0)
    ring = torch.empty(nb.nvbt_channel_bytes(1000), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring)
    dr.run_stencil(ctx, nb.TOOL_TRACE, buf0, buf1, n, iters)
    d = nb.nvbt_channel_drain_digest(ch, timeout_us=60_000_000)
    acc = ev.Accumulator(programs.stencil(), trace=True)
    m_st.run_iterations(acc, n, buf0.data_ptr(), buf1.data_ptr(), iters)
    assert (d.n_rec, d.d1, d.d2) == (acc.digest.n, acc.digest.d1, acc.digest.d2)


# ---------------------------------------------------------------- F2 device-memory channel + GPU consumer
def _device_ring(nb, ctx, records):
    import torch
    ring = torch.empty(64 + 288 * records, dtype=torch.uint8, device="cuda")
    ring.view(torch.int32).fill_(1)            # stale "committed" tags everywhere: open must clear them
    return ring, nb.nvbt_channel_open(ctx, ring)


def _committed(ring):
    """Records of a device ring with tag 1 (slots are spread over SM regions), tag word cleared."""
    r = ring[64:].cpu().numpy().reshape(-1, 288)
    r = r[r[:, 28:32].copy().view("<u4")[:, 0] == 1].copy()
    r[:, 28:32] = 0
    return r


@pytest.mark.parametrize("n,iters,slots", [(96, 3, 64), (100, 2, 64), (512, 16, 128)])
def test_device_channel_footprint_stencil(nvbt, n, iters, slots):
    """F2: records stay in HBM and the GPU consumer's per-launch footprint equals the oracle's; the
    records themselves (copied back only for the check) equal the oracle's as a multiset."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.TRACE)
    x0 = cuda(uniform_f32((n, n), 4))
    buf0, buf1 = x0.clone(), torch.zeros_like(x0)
    ring, ch = _device_ring(nb, ctx, 1 << 21)
    dr.run_stencil(ctx, nb.TOOL_TRACE, buf0, buf1, n, iters)
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    m_st.run_iterations(acc, n, buf0.data_ptr(), buf1.data_ptr(), iters)
    exp = acc.record_array()
    fp = nb.nvbt_trace_footprint(ch, iters + 1, table_slots=slots)   # 512x16: crowded table
    assert np.array_equal(fp.astype(np.int64), trace.footprint(exp, iters + 1))
    assert nb.nvbt_channel_dropped(ch) == 0
    got = _committed(ring)
    assert len(got) == len(exp)
    assert (trace.sort_records(got) == trace.sort_records(exp)).all()
    with pytest.raises(nb.NvbtError):
        nb.nvbt_channel_drain_digest(ch, timeout_us=1000)


def test_device_channel_overflow_drops(nvbt):
    """A device ring smaller than the trace keeps what fits and counts the rest as dropped (no
    backpressure wait: nobody frees slots); every kept record is one of the oracle's and the consumer
    counts exactly the kept ones. A table too small for the footprint is an error, not a hang."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n, iters, cap = 64, 2, 1000
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.TRACE)
    buf0 = cuda(uniform_f32((n, n), 4)); buf1 = torch.zeros_like(buf0)
    ring, ch = _device_ring(nb, ctx, cap)
    dr.run_stencil(ctx, nb.TOOL_TRACE, buf0, buf1, n, iters)
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    m_st.run_iterations(acc, n, buf0.data_ptr(), buf1.data_ptr(), iters)
    exp = acc.record_array()
    fp = nb.nvbt_trace_footprint(ch, iters, table_slots=1 << 6)
    got = _committed(ring)
    assert 0 < len(got) <= cap
    assert int(fp[:, 2].sum()) == len(got)
    assert nb.nvbt_channel_dropped(ch) == len(exp) - len(got)
    universe = {r.tobytes() for r in exp}
    assert all(r.tobytes() in universe for r in got)
    assert len({r.tobytes() for r in got}) == len(got)
    with pytest.raises(nb.NvbtError):                      # 1 slot < 2 launches x regions: reported, no hang
        nb.nvbt_trace_footprint(ch, iters, table_slots=1)


def test_device_channel_footprint_bfs(nvbt):
    """F2 on the irregular workload: BFS (two kernels per level) on an R-MAT graph."""
    nb, dr = nvbt.nvbt, nvbt.drivers
    rowptr, col = rmat_csr(10)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    ctx = nb.nvbt_init(nb.W_BFS, nb.TRACE)
    rp, cl = cuda(rowptr), cuda(col)
    bufs = dr.bfs_buffers(n, "cuda")
    ring, ch = _device_ring(nb, ctx, 1 << 20)
    cost, levels = dr.run_bfs(ctx, nb.TOOL_TRACE, rp, cl, src, bufs)
    acc = ev.Accumulator(programs.bfs(), trace=True, keep_records=True)
    ptr = m_bfs.Ptrs(bufs["mask"].data_ptr(), bufs["visited"].data_ptr(), bufs["updating"].data_ptr(),
                     bufs["cost"].data_ptr(), bufs["over"].data_ptr(), rp.data_ptr(), cl.data_ptr())
    m_bfs.run(acc, rowptr, col, src, ptr)
    exp = acc.record_array()
    nl = int(exp.view(trace.RECORD_DTYPE)["launch"].max()) + 1
    fp = nb.nvbt_trace_footprint(ch, nl, table_slots=1 << 12)
    assert nb.nvbt_channel_dropped(ch) == 0
    assert np.array_equal(fp.astype(np.int64), trace.footprint(exp, nl))


# ---------------------------------------------------------------- C5 generator + replay
def test_generator_bytes_match_oracle(nvbt):
    import torch
    nb = nvbt.nvbt
    ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT)
    for first, n in [(0, 1 << 16), (10**10 - 4099, 4099)]:
        hdr = torch.zeros(n * 16, dtype=torch.uint8, device="cuda")
        addr = torch.zeros(n * 256, dtype=torch.uint8, device="cuda")
        nb.nvbt_gen_events(ctx, gen.SEED, first, n, hdr, addr)
        pc, warp, A, P, oaddr = gen.events(first, n)
        h = hdr.cpu().numpy().view("<u4").reshape(n, 4)
        assert (h[:, 0] == pc).all() and (h[:, 1] == warp).all() and (h[:, 2] == A).all() and (h[:, 3] == P).all()
        ga = addr.cpu().numpy().view("<u8").reshape(n, 32)
        assert (ga == oaddr).all()   # non-memory slots are not written by either side (zeros here)


# "staged" = nvbt_replay_staged (two passes, scratch list; "staged-small": a few thousand events per
# block, so one call runs several pass pairs); "single" = the single-pass nvbt_replay
REPLAY_VARIANTS = ["staged", "staged-small", "single"]


def _replay_scratch(nb, ctx, variant, monkeypatch):
    """Scratch tensor for the staged variants, None for the single pass."""
    import torch
    if not variant.startswith("staged"):
        return None
    per = 5000 if variant == "staged-small" else 1 << 20
    return torch.empty(nb.nvbt_replay_scratch_size(ctx, per), dtype=torch.uint8, device="cuda")


@pytest.mark.parametrize("variant", REPLAY_VARIANTS)
@pytest.mark.parametrize("first,n", [(0, 1 << 18), (123456789, 100_003)])
def test_replay_parity(nvbt, first, n, variant, monkeypatch):
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=1 << 20)
    scratch = _replay_scratch(nb, ctx, variant, monkeypatch)
    chunk = 1 << 16
    hdr = torch.empty(chunk * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty(chunk * 256, dtype=torch.uint8, device="cuda")
    dr.replay_range(ctx, gen.SEED, first, n, hdr, addr, scratch=scratch)
    g = read_all(nb, ctx, per_warp=True)
    acc = ev.Accumulator(programs.replay(), n_warps=1 << 20)
    gen.replay(acc, first, n)
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS + ["PW_T", "PW_W"], f"replay [{first}, +{n})")
    assert nb.nvbt_replay_errors(ctx) == 0


@pytest.mark.parametrize("staged", [False, True])
def test_replay_merge_equals_single(nvbt, staged):
    """a8: three partitions merged by summing the packed accumulator region equal one run (I-6); the
    single run uses the other replay path, so the two paths also agree with each other."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    n = 200_000
    hdr = torch.empty((1 << 16) * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty((1 << 16) * 256, dtype=torch.uint8, device="cuda")
    whole = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    scratch = torch.empty(nb.nvbt_replay_scratch_size(whole, 1 << 16), dtype=torch.uint8, device="cuda")
    dr.replay_range(whole, gen.SEED, 0, n, hdr, addr, scratch=None if staged else scratch)
    parts = []
    for r in range(3):
        lo, hi = dr.shard_range(n, r, 3)
        c = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
        dr.replay_range(c, gen.SEED, lo, hi - lo, hdr, addr, scratch=scratch if staged else None)
        parts.append(c)
    v0 = nb.nvbt_accum_view(parts[0])
    v0 += nb.nvbt_accum_view(parts[1]) + nb.nvbt_accum_view(parts[2])
    torch.cuda.synchronize()
    assert torch.equal(nb.nvbt_accum_view(parts[0]), nb.nvbt_accum_view(whole))
    assert_same(read_all(nb, parts[0]), read_all(nb, whole), what="merged replay")


def _adversarial_stream(n, seed):
    """Handcrafted replay events stressing every sectors_lines() path: monotone runs, 32 KB bitmap window
    edges (incl. keys below the first lane), 32-bit relative sort, 64-bit sort, partial and sparse masks,
    duplicate sectors, line-boundary straddles, widths 1..16; wide rows (upper address words differ) with
    repeated addresses and with lines shared by lane pairs (the hashed all-distinct test must fail them and
    the exact fallback count them)."""
    rng = np.random.default_rng(seed)
    prog = programs.replay()
    mem_pcs = np.nonzero(programs.is_mem(prog))[0]
    pc = rng.choice(mem_pcs, size=n)
    warp = rng.integers(0, 1 << 20, size=n)
    A = rng.integers(1, 1 << 32, size=n, dtype=np.uint64).astype(np.uint32)
    A[: n // 2] = 0xFFFFFFFF
    P = np.where(rng.random(n) < 0.5, np.uint32(0xFFFFFFFF),
                 rng.integers(0, 1 << 32, size=n, dtype=np.uint64).astype(np.uint32))
    lane = np.arange(32, dtype=np.int64)[None, :]
    base = (rng.integers(1 << 20, 1 << 40, size=(n, 1)) & ~127).astype(np.int64)
    kind = rng.integers(0, 10, size=(n, 1))
    span = rng.choice([32, 1024 * 32 - 1, 1024 * 32, 1024 * 32 + 32, 1 << 20, 1 << 38], size=(n, 1))
    r = rng.integers(0, 1 << 62, size=(n, 32)) % span - span // 2       # symmetric around base
    stride = rng.choice([0, 1, 4, 8, 16, 31, 32, 33, 64, 127, 128, 129, 4096, 1 << 20], size=(n, 1))
    off = rng.integers(0, 4096, size=(n, 1))                            # unaligned progression starts
    hb = ((base >> 32) + 1) << 32                                       # next 4 GB boundary
    addr = np.select([kind == 0, kind == 1, kind == 2, kind == 3, kind == 4, kind == 5, kind == 6],
                     [base + off + lane * stride,                         # monotone / arithmetic progression
                      base - lane * stride,                               # decreasing
                      base + (r // 4) * 4,                                # window / wide random
                      base + (lane % 3) * 32 + 124,                       # duplicates straddling lines
                      base + r[:, (lane[0] * 7) % 8],                     # wide random with repeats
                      hb - 8 * stride + lane * stride,                    # progression across a 4 GB line
                      base + (lane % 2) * 32 + (lane // 2) * (1 << 33)],  # lines shared by lane pairs, 4 GB apart
                     base + r)
    addr = np.clip(addr, 0, (1 << 62) - 1).astype(np.uint64)
    return pc.astype(np.int64), warp.astype(np.int64), A, P, addr


@pytest.mark.parametrize("variant", REPLAY_VARIANTS)
@pytest.mark.parametrize("seed", [1, 2])
def test_replay_adversarial_addresses(nvbt, seed, variant, monkeypatch):
    import torch
    nb = nvbt.nvbt
    n = 40_000
    pc, warp, A, P, addr = _adversarial_stream(n, seed)
    hdr = gen.header_bytes(pc, warp, A, P)
    ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    scratch = _replay_scratch(nb, ctx, variant, monkeypatch)
    d_hdr = cuda(hdr.view(np.uint8).reshape(-1))
    d_addr = cuda(addr.view(np.uint8).reshape(-1))
    if scratch is None:
        nb.nvbt_replay(ctx, d_hdr, d_addr, n)
    else:
        nb.nvbt_replay_staged(ctx, d_hdr, d_addr, n, scratch)
    g = read_all(nb, ctx)
    acc = ev.Accumulator(programs.replay())
    acc.add(0, warp, pc, A, P, addr)
    assert_same(g, acc.result(), COUNT_KEYS + MEM_KEYS, f"adversarial replay seed {seed}")


# ---------------------------------------------------------------- degenerate cases
def test_degenerate_shapes(nvbt):
    """Empty launches, single-element grids, all-boundary stencils, isolated BFS sources."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    # vectorAdd N = 0 launches nothing and counts nothing; N = 1 is a single live lane
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.MEMDIV)
    a = cuda(uniform_f32(1, 1))
    c = torch.empty_like(a)
    nb.nvbt_vectoradd(ctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV, a, a, c, 0)
    assert (nb.nvbt_count(ctx) == 0).all()
    nb.nvbt_vectoradd(ctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV, a, a, c, 1)
    acc = ev.Accumulator(programs.vectoradd())
    m_va.run(acc, 1, a.data_ptr(), a.data_ptr(), c.data_ptr())
    assert_same(read_all(nb, ctx), acc.result(), COUNT_KEYS + MEM_KEYS, "vectorAdd N=1")
    # SGEMM 1x1x1
    ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.MEMDIV)
    A = cuda(np.ones((1, 1), np.float32))
    Cm = torch.empty(1, 1, device="cuda")
    nb.nvbt_sgemm(ctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV, A, A, Cm, 1, 1, 1)
    acc = ev.Accumulator(programs.sgemm())
    m_sg.run(acc, 1, 1, 1, A.data_ptr(), A.data_ptr(), Cm.data_ptr())
    assert_same(read_all(nb, ctx), acc.result(), COUNT_KEYS + MEM_KEYS, "SGEMM 1x1x1")
    # stencil n = 2: every point is a boundary point (P1 false everywhere)
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.MEMDIV)
    x = cuda(uniform_f32((2, 2), 4))
    y = torch.zeros_like(x)
    nb.nvbt_stencil(ctx, nb.TOOL_COUNT | nb.TOOL_MEMDIV, x, y, 2)
    acc = ev.Accumulator(programs.stencil())
    m_st.run(acc, 2, x.data_ptr(), y.data_ptr())
    assert_same(read_all(nb, ctx), acc.result(), COUNT_KEYS + MEM_KEYS, "stencil n=2")
    assert torch.equal(y, x)
    # BFS from an isolated vertex: one level, nothing reached
    rowptr = np.array([0, 0, 1, 2], dtype=np.int32)
    col = np.array([2, 1], dtype=np.int32)
    ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB | nb.MEMDIV)
    rp, cl = cuda(rowptr), cuda(col)
    bufs = dr.bfs_buffers(3, "cuda")
    cost, levels = dr.run_bfs(ctx, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV, rp, cl, 0, bufs)
    acc = ev.Accumulator(programs.bfs())
    ptr = m_bfs.Ptrs(bufs["mask"].data_ptr(), bufs["visited"].data_ptr(), bufs["updating"].data_ptr(),
                     bufs["cost"].data_ptr(), bufs["over"].data_ptr(), rp.data_ptr(), cl.data_ptr())
    ocost, olevels, _ = m_bfs.run(acc, rowptr, col, 0, ptr)
    assert levels == olevels == 1 and cost.cpu().tolist() == ocost.tolist() == [0, -1, -1]
    assert_same(read_all(nb, ctx), acc.result(), COUNT_KEYS + MEM_KEYS, "BFS isolated source")
    # replay of zero events is a no-op; an out-of-range pc is counted as an error and ignored
    rctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    h = np.zeros((2, 4), dtype="<u4")
    h[0] = [5, 1, 0xFFFFFFFF, 0xFFFFFFFF]
    h[1] = [4096 + 7, 1, 0xFFFFFFFF, 0xFFFFFFFF]
    d_h = cuda(h.view(np.uint8).reshape(-1))
    d_a = torch.zeros(2 * 256, dtype=torch.uint8, device="cuda")
    nb.nvbt_replay(rctx, d_h, d_a, 0)
    assert (nb.nvbt_count(rctx) == 0).all()
    nb.nvbt_replay(rctx, d_h, d_a, 2)
    assert nb.nvbt_replay_errors(rctx) == 1
    assert nb.nvbt_count(rctx).tolist() == [32, 32, 1, 1]
    # the staged replay: same degenerate behaviour, and a scratch too small for one block is ENOMEM
    sctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.MEMDIV)
    scratch = torch.empty(nb.nvbt_replay_scratch_size(sctx, 1), dtype=torch.uint8, device="cuda")
    nb.nvbt_replay_staged(sctx, d_h, d_a, 0, scratch)
    assert (nb.nvbt_count(sctx) == 0).all()
    nb.nvbt_replay_staged(sctx, d_h, d_a, 2, scratch)
    assert nb.nvbt_replay_errors(sctx) == 1
    assert nb.nvbt_count(sctx).tolist() == [32, 32, 1, 1]
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_replay_staged(sctx, d_h, d_a, 2, scratch[: scratch.numel() // 2])
    assert e.value.code == nb.ENOMEM
    cctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT)        # no MEMDIV: no list, scratch may be None
    nb.nvbt_replay_staged(cctx, d_h, d_a, 2, None)
    assert nb.nvbt_count(cctx).tolist() == [32, 32, 1, 1]


def test_api_errors(nvbt):
    """Argument validation surfaces as NvbtError with the documented codes."""
    import torch
    nb = nvbt.nvbt
    ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT)
    x = torch.zeros(64, device="cuda")
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_sgemm(ctx, nb.TOOL_COUNT | nb.TOOL_BBCOUNT, x, x, x, 4, 4, 4)
    assert e.value.code == nb.EINVAL
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_sgemm(ctx, nb.TOOL_COUNT, x, x, x, 4, 4, 0)          # K >= 1
    assert e.value.code == nb.EINVAL
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_sgemm(ctx, nb.TOOL_TRACE, x, x, x, 4, 4, 4)          # TRACE not enabled
    assert e.value.code == nb.ESTATE
    ring = torch.empty(4096, dtype=torch.uint8)                       # not pinned
    tctx = nb.nvbt_init(nb.W_STENCIL, nb.TRACE)
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_channel_open(tctx, ring)
    assert e.value.code == nb.EINVAL


# ---------------------------------------------------------------- F1 kernel sampling
class PerLaunch:
    """Oracle accumulator that keeps one numpy Accumulator per launch id (to form F1's extrapolation
    from the oracle's own per-launch results)."""

    def __init__(self, prog):
        self.prog, self.by_launch = prog, {}

    def add(self, launch, *a, **kw):
        self.by_launch.setdefault(launch, ev.Accumulator(self.prog)).add(launch, *a, **kw)

    def result(self, launches=None, factor=1):
        ks = sorted(self.by_launch) if launches is None else launches
        out = None
        for k in ks:
            r = self.by_launch[k].result()
            r.pop("trace")
            out = r if out is None else {x: out[x] + r[x] for x in out}
        return {x: v * factor for x, v in out.items()}


def test_kernel_sampling_exact_when_control_flow_is_grid_only(nvbt):
    """"If the control flow of a kernel does not change based on the values computed, but it is
    only a function of the grid dimensions, the sampling error is 0%" — stencil and vectorAdd qualify:
    the sampled estimate equals the ORACLE's full run (every launch modelled) element by element, and so
    does the fully instrumented GPU run."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV
    tools = nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV
    # stencil: 2 grid shapes over 3 runs (ping-pong buffers: the addresses alternate between launches,
    # but every launch of a shape has the same S/L per event, so the extrapolation is still exact)
    full = nb.nvbt_init(nb.W_STENCIL, flags)
    samp = nb.nvbt_init(nb.W_STENCIL, flags)
    scratch = nb.nvbt_init(nb.W_STENCIL, flags)
    sampler = dr.KernelSampler(samp, scratch)
    acc = ev.Accumulator(programs.stencil())
    launch = 0
    for n, iters in [(96, 5), (64, 3), (96, 2)]:
        x0 = cuda(uniform_f32((n, n), 4))
        b0, b1 = x0.clone(), torch.zeros_like(x0)
        m_st.run_iterations(acc, n, b0.data_ptr(), b1.data_ptr(), iters, first_launch=launch)
        launch += iters
        bufs = (b0, b1)
        for it in range(iters):
            src, dst = bufs[it % 2], bufs[(it + 1) % 2]
            nb.nvbt_stencil(full, tools, src, dst, n)
            sampler.launch(("stencil", n), lambda c, t: nb.nvbt_stencil(c, t, src, dst, n), tools)
    launches = sampler.finish()
    assert launches == {("stencil", 96): 7, ("stencil", 64): 3}
    ref = acc.result()
    assert_same(read_all(nb, samp), ref, COUNT_KEYS + MEM_KEYS, "sampled stencil vs oracle full run")
    assert_same(read_all(nb, full), ref, COUNT_KEYS + MEM_KEYS, "full stencil vs oracle")
    # vectorAdd: 3 sizes (one ragged), 4 launches each
    samp = nb.nvbt_init(nb.W_VECTORADD, flags)
    scratch = nb.nvbt_init(nb.W_VECTORADD, flags)
    sampler = dr.KernelSampler(samp, scratch)
    acc = ev.Accumulator(programs.vectoradd())
    for N in (4096, 1000, 65536):
        a, b = cuda(uniform_f32(N, 1)), cuda(uniform_f32(N, 2))
        c = torch.empty_like(a)
        for _ in range(4):
            m_va.run(acc, N, a.data_ptr(), b.data_ptr(), c.data_ptr())
            sampler.launch(("vectoradd", N), lambda cx, t: nb.nvbt_vectoradd(cx, t, a, b, c, N), tools)
    sampler.finish()
    assert_same(read_all(nb, samp), acc.result(), COUNT_KEYS + MEM_KEYS, "sampled vectorAdd vs oracle")


def test_kernel_sampling_error_on_data_dependent_kernels(nvbt):
    """BFS levels share grid dimensions but not control flow, so sampling (one instrumented level, its
    counts extrapolated to every level) has an error, stated against the ORACLE's exact counts: the GPU's
    sampled estimate equals levels x the oracle's level-0 counts element by element, the GPU's full run
    equals the oracle's exact counts, and the relative error of W_issued is their quotient."""
    import torch
    nb, dr = nvbt.nvbt, nvbt.drivers
    rowptr, col = rmat_csr(10, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    rp, cl = cuda(rowptr), cuda(col)
    full = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    dr.run_bfs(full, nb.TOOL_BBCOUNT, rp, cl, src)
    samp = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    scratch = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    sampler = dr.KernelSampler(samp, scratch)
    bufs = dr.bfs_buffers(n, "cuda")
    bufs["mask"][src] = 1; bufs["visited"][src] = 1; bufs["cost"][src] = 0
    level = 0
    while True:
        bufs["over"].zero_(); bufs["updating"].zero_()
        sampler.launch(("bfs", n), lambda c, t: nb.nvbt_bfs_level(c, t, rp, cl, n, bufs["mask"], bufs["visited"],
                                                                  bufs["updating"], bufs["cost"], bufs["over"],
                                                                  level),
                       nb.TOOL_BBCOUNT)
        torch.cuda.synchronize()
        level += 1
        if int(bufs["over"].item()) == 0:
            break
    sampler.finish()
    per = PerLaunch(programs.bfs())
    _, olevels, _ = m_bfs.run(per, rowptr, col, src, m_bfs.Ptrs(*([1 << 32] * 7)))
    assert olevels == level
    exact = per.result()
    est = per.result(launches=[0, 1], factor=level)          # level 0 = launches 0 (expand) and 1 (update)
    assert_same(read_all(nb, full), exact, COUNT_KEYS, "full BFS vs oracle")
    assert_same(read_all(nb, samp), est, COUNT_KEYS, "sampled BFS vs oracle extrapolation")
    err = abs(int(est["counts"][2]) - int(exact["counts"][2])) / int(exact["counts"][2])
    assert err > 0.0                                         # not exact: control flow depends on data
    print(f"F1 BFS scale 10: {level} levels, W_issued exact {int(exact['counts'][2])}, "
          f"sampled {int(est['counts'][2])}, relative error {err:.4f}")
