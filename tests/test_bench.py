"""bench.py's contract (one JSON line; the driver's keys) at reduced sizes.

CPU: the reference arm (the C oracle on the host cores). GPU: the default line with every config beside
the C2 headline, and `--gpus 2` without torchrun (it re-launches itself under torch.distributed.run) on
one GPU over gloo — the N > 1 path: CTA-row partition of C1/C2, partitioned BFS with its MAX exchanges,
row-slab stencil with P2P halos and a channel per rank, event ranges for C5, the int64 merge, and the
closed-form checks on the merged counters."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SMALL = ["--bfs-scale", "14", "--stencil-n", "1024", "--stencil-iters", "4", "--replay-events", "300000000",
         "--ring-records", "65536"]


def run_bench(args, env=None, timeout=900):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       cwd=ROOT, env=e, timeout=timeout)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = run_bench(["--impl", "reference", "--steps", "1", "--warmup", "3"])
    assert d["impl"] == "reference" and d["unit"] == "events/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == len(os.sched_getaffinity(0))
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


@pytest.mark.gpu
def test_bench_line_all_configs(nvbt):
    d = run_bench(["--steps", "3", "--warmup", "3", *SMALL])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["counts_check"] == "ok" and d["gpu_launches"] == 3
    assert d["cpu_baseline"]["matches_gpu"] is True
    assert set(d["configs"]) == {"c1", "c3", "c4", "c4_compact", "c4_line", "c5"}
    for name, c in d["configs"].items():
        assert c["counts_check"].startswith("ok"), (name, c["counts_check"])
        assert c["value"] > 0


@pytest.mark.gpu
def test_bench_two_ranks_gloo_same_gpu(nvbt):
    d = run_bench(["--gpus", "2", "--steps", "3", "--warmup", "3", *SMALL],
                  env={"NVBT_BENCH_BACKEND": "gloo", "NVBT_BENCH_SAME_GPU": "1"})
    assert d["n_gpus"] == 2 and d["counts_check"] == "ok" and d["scaling"] == "strong"
    assert "CTA-row partition" in d["config"]["parallelism"]
    for name, c in d["configs"].items():
        assert c["counts_check"].startswith("ok"), (name, c["counts_check"])
    assert set(d["allreduce_latency"]) == {"8KiB_us", "64KiB_us", "1024KiB_us"}
