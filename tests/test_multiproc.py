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
