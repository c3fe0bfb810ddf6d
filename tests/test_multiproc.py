"""N > 1 host logic on CPU with the gloo backend, world size 2: event-range sharding,
the int64 SUM merge of packed accumulators (a8), and the max-over-ranks timing reduction of bench.py.
The per-rank partial results come from the oracle, so the merged result must equal the single-process
oracle result exactly (partition invariance, I-6)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

KEYS = ["counts", "H_t", "H_w", "Ent_t", "Ent_w", "Ins_t", "Ins_w", "mem_n", "mem_S", "mem_L", "hS", "hL"]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def pack(r):
    return torch.from_numpy(np.concatenate([np.asarray(r[k], dtype=np.int64) for k in KEYS]))


def _worker(rank, world, port, n, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_micro_villasnk19_b200 import drivers
        from oracle import events as ev, programs, gen
        import bench
        lo, hi = drivers.shard_range(n, rank, world)
        acc = ev.Accumulator(programs.replay())
        gen.replay(acc, lo, hi - lo)
        t = pack(acc.result())
        drivers.merge_tensor(t)
        tmax = bench.max_over_ranks(float(rank + 1), world)
        tsum = bench.sum_over_ranks(float(hi - lo), world)
        if rank == 0:
            out_q.put((t.numpy(), tmax, tsum))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n", [6001, 64])
def test_gloo_merge_equals_single_process(n):
    from oracle import events as ev, programs, gen
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, q)) for r in range(2)]
    for p in procs:
        p.start()
    merged, tmax, tsum = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    acc = ev.Accumulator(programs.replay())
    gen.replay(acc, 0, n)
    assert (merged == pack(acc.result()).numpy()).all()
    assert tmax == 2.0 and tsum == float(n)


def test_shard_range_partitions_exactly():
    from paper_conf_micro_villasnk19_b200 import drivers
    for n in (0, 1, 7, 10**10 + 3):
        for world in (1, 2, 3, 8):
            parts = [drivers.shard_range(n, r, world) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[i][1] == parts[i + 1][0] for i in range(world - 1))
            assert max(h - l for l, h in parts) - min(h - l for l, h in parts) <= 1


def test_merge_rejects_non_int64():
    from paper_conf_micro_villasnk19_b200 import drivers
    with pytest.raises(TypeError):
        drivers.merge_tensor(torch.zeros(3, dtype=torch.float32))


def _halo_worker(rank, world, port, n, out_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_micro_villasnk19_b200 import drivers
        # every rank's buffer: its own rows carry (rank, row, col)-dependent values, all others garbage
        g = torch.full((n, n), -7.0)
        r0, r1 = drivers.stencil_rows(n, rank, world)
        rows = torch.arange(n, dtype=torch.float32)[:, None] * 1000 + torch.arange(n, dtype=torch.float32)[None, :]
        g[r0:r1] = rows[r0:r1] + 0.5
        drivers._exchange_halo(g, n, rank, world, None)
        out_q.put((rank, r0, r1, g.numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,world", [(50, 3), (64, 2), (17, 4)])
def test_gloo_stencil_halo_exchange(n, world):
    """C4 partition: after the exchange every rank holds the true row just above and just
    below its slab (P2P send/recv with the nearest non-empty slabs, including across a rank whose slab is
    empty: n = 17 has 3 CTA rows for 4 ranks); nothing else changes."""
    from paper_conf_micro_villasnk19_b200 import drivers
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    rows = np.arange(n, dtype=np.float32)[:, None] * 1000 + np.arange(n, dtype=np.float32)[None, :] + 0.5
    covered = np.zeros(n, dtype=int)
    for rank, r0, r1, g in res:
        covered[r0:r1] += 1
        expect = np.full((n, n), -7.0, dtype=np.float32)
        expect[r0:r1] = rows[r0:r1]
        if r1 > r0:
            if r0 > 0:
                expect[r0 - 1] = rows[r0 - 1]
            if r1 < n:
                expect[r1] = rows[r1]
        assert np.array_equal(g, expect), rank
    assert (covered == 1).all()                  # the slabs partition the grid


def test_cta_rows_partition():
    from paper_conf_micro_villasnk19_b200 import drivers
    for gy in (1, 2, 7, 1024):
        for world in (1, 2, 3, 8):
            parts = [drivers.cta_rows(gy, r, world) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == gy
            assert all(parts[i][1] == parts[i + 1][0] for i in range(world - 1))
