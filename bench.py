#!/usr/bin/env python
"""nvbt benchmark: instrumented warp-instruction events/s and slowdown vs the uninstrumented kernel
(BASELINE.json metric), on all five BASELINE.json configs.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--configs c1,c3,c4,c5]

One JSON line. `value` is the headline config C2 (configs[1]: naive row-fastest SGEMM 1024^3 with the
bench tool set BBCOUNT|MEMDIV: counts, opcode/BB histograms via basic-block-entry hooks, per-instruction
memory divergence), one step = one instrumented launch; `configs` holds the other four configs measured in
the same run (C1 vectorAdd, C3 BFS on R-MAT scale 20, C4 the 8192^2 x 100 stencil traced through the
pinned-host channel, C5 the replay of 10^10 generated events), each with its value, slowdown, roofline
fraction and a result check.

Multi-GPU: one process per GPU. Without torchrun, `--gpus N` (N > 1) re-launches itself
under torch.distributed.run. Work is partitioned, total work fixed ("strong"): C1/C2 by CTA rows of the
same launch (nvbt_set_partition), C3 by vertex range with its per-level MAX exchanges, C4 by row slab with
P2P halos and one channel per rank, C5 by event-index range; the per-GPU counters are merged by one int64
SUM all-reduce (a8) and checked against the closed forms. Timing: CUDA events on the launching stream,
max over ranks; L2 flushed (256 MiB write) between C2 steps; clocks sampled with nvidia-smi during the
timed region.

`--impl reference`: the reference arm of this tier is the CPU oracle: the multithreaded C
oracle (oracle/c) on all host cores, one whole C2 launch per step.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}
N_SM = 148
METRIC = "instrumented warp-instr events/sec and slowdown vs uninstrumented"
SEED = 0x4E5642544E564254


def _profile_json(name):
    try:
        with open(os.path.join(ROOT, "profiles", name)) as f:
            return json.load(f)
    except Exception:
        return None


def load_traffic(kernel):
    """DRAM bytes per launch of `kernel` from the committed ncu capture (profiles/r2_traffic.json)."""
    d = _profile_json("r2_traffic.json")
    return None if d is None else d.get(kernel)


def load_counters(kernel, keys=("warp_inst_per_unit", "dram_bytes_per_unit", "shared_atomic_wavefronts_per_unit",
                                 "global_atomic_sectors_per_unit", "issue_active_pct")):
    """ncu counters per unit of work of `kernel` from the committed capture (profiles/r2_ncu_counters.json)."""
    d = (_profile_json("r2_ncu_counters.json") or {}).get(kernel)
    return None if d is None else {k: d[k] for k in keys if k in d}


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return PEAKS_FALLBACK, "fallback (B200_PROFILING.md)"


def d2h_peak():
    """Measured SM-store bandwidth into pinned host memory (tools/peaks/peaks.cu, profiles/r1_box_peaks.json)."""
    d = _profile_json("r1_box_peaks.json") or {}
    return float(d.get("sm_store16_host_GBs_occ4", 52.7))


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


# --------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits", "-lms", "100",
                 "-i", str(self.gpu)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thr = threading.Thread(target=self._read, daemon=True)
            self.thr.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if len(r) > 5 + k and r[5 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# --------------------------------------------------------------------------- distributed
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def spawn_ranks(n):
    """`--gpus N` without torchrun: re-launch this script under torch.distributed.run (one rank per GPU)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__),
           *sys.argv[1:]]
    return subprocess.call(cmd)


HOST_PLACEMENT = None   # set by dist_setup for N > 1: the rank's host CPUs (NUMA-local drain)


def dist_setup(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("NVBT_BENCH_SAME_GPU"):   # test hook: all ranks on GPU 0 (with a gloo backend)
        local = 0
    torch.cuda.set_device(local)
    global HOST_PLACEMENT
    if world > 1 and not os.environ.get("NVBT_BENCH_SAME_GPU") and os.environ.get("NVBT_BENCH_NUMA", "1") != "0":
        # the rank's drain threads and pinned ring on its GPU's NUMA node, the node's cores split between
        # the ranks sharing it (before any pinned allocation and before the drain pool exists)
        from paper_conf_micro_villasnk19_b200 import drivers
        cpus = drivers.bind_rank_to_gpu_numa(local)
        HOST_PLACEMENT = {"numa_local": cpus is not None, "cpus": len(cpus) if cpus else len(os.sched_getaffinity(0))}
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("NCCL_DEBUG", "INFO")          # communicator init log (ranks, NVLS, channels)
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        backend = os.environ.get("NVBT_BENCH_BACKEND", "nccl")
        kw = {"device_id": torch.device("cuda", local)} if backend == "nccl" else {}
        dist.init_process_group(backend, **kw)
    return rank, world, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def _reduce(x, world, op):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=op)
    return float(t.item())


def max_over_ranks(x, world, device=None):
    import torch.distributed as dist
    return _reduce(x, world, dist.ReduceOp.MAX if world > 1 else None)


def sum_over_ranks(x, world, device=None):
    import torch.distributed as dist
    return _reduce(x, world, dist.ReduceOp.SUM if world > 1 else None)


def merge(dr, ctx, world):
    """a8: one int64 SUM all-reduce of the packed accumulator region (after the timed region)."""
    if world > 1:
        dr.merge(ctx)


def allreduce_latency(world):
    """int64 SUM all-reduce latency of 8 KB / 64 KB / 1 MB messages (the merge's
    sizes), median of 20 after 5 warm-ups, device-timed, max over ranks."""
    import torch
    import torch.distributed as dist
    out = {}
    for nbytes in (8 << 10, 64 << 10, 1 << 20):
        t = torch.zeros(nbytes // 8, dtype=torch.int64, device="cuda")
        for _ in range(5):
            dist.all_reduce(t)
        ts = []
        for _ in range(20):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dist.all_reduce(t)
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        out[f"{nbytes >> 10}KiB_us"] = max_over_ranks(statistics.median(ts), world)
    return out


def timed_steps(torch, fn, n, flush=None):
    """n steps, each bracketed by CUDA events on the current stream (the contexts' stream)."""
    ts = []
    for _ in range(n):
        if flush is not None:
            flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    return ts


def _timed_events(torch, fn, n):
    return timed_steps(torch, fn, n)


# --------------------------------------------------------------------------- C2 SGEMM (headline)
# hook instruction minima per event used for the issue roofline (minimal SASS per hook)
HOOK_OPS = {"count": 4, "guard": 6, "mem": 23}


class SgemmBench:
    name = "c2"
    M = N = K = 1024
    desc = ("C2 naive row-fastest SGEMM 1024^3 (fp32), tools BBCOUNT|MEMDIV (counts, opcode+BB histograms via "
            "BB-entry hooks, per-instruction divergence)")

    def __init__(self, torch, nb, dr, rank, world):
        self.torch, self.nb, self.dr = torch, nb, dr
        from synth import uniform_f32
        M, N, K = self.M, self.N, self.K
        self.nw = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
        self.ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)
        if world > 1:   # this rank runs CTA rows [y0, y1) of the one 1024^3 launch
            nb.nvbt_set_partition(self.ctx, rank, world)
        gx, gy = -(-M // 32), -(-N // 8)
        y0, y1 = dr.cta_rows(gy, rank, world)
        self.rank_warps = (y1 - y0) * gx * 8
        self.tools = nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV
        self.hA = torch.from_numpy(uniform_f32((M, K), 3, -1, 1)).pin_memory()
        self.hB = torch.from_numpy(uniform_f32((K, N), 4, -1, 1)).pin_memory()
        self.A, self.B = self.hA.cuda(), self.hB.cuda()
        self.C = torch.empty(M, N, device="cuda")
        # events per launch (EM §3.2): every warp runs 12 + 6K warp-level instructions
        self.per_warp = 12 + 6 * K
        self.events = self.nw * self.per_warp
        self.launched = 0

    def plain(self):
        self.nb.nvbt_sgemm(self.ctx, self.nb.TOOL_NONE, self.A, self.B, self.C, self.M, self.N, self.K)

    def instr(self):
        self.nb.nvbt_sgemm(self.ctx, self.tools, self.A, self.B, self.C, self.M, self.N, self.K)
        self.launched += 1

    def reset(self):
        self.nb.nvbt_reset(self.ctx)
        self.launched = 0   # instrumented launches accumulated in the context since the reset

    def e2e_step(self, out_host):
        """Through the public API with host buffers: H2D inputs, instrumented launch, read results."""
        nb = self.nb
        self.A.copy_(self.hA, non_blocking=True)
        self.B.copy_(self.hB, non_blocking=True)
        nb.nvbt_sgemm(self.ctx, self.tools, self.A, self.B, self.C, self.M, self.N, self.K)
        self.launched += 1
        out_host["counts"] = nb.nvbt_count(self.ctx)
        out_host["memdiv"] = nb.nvbt_mem_divergence(self.ctx)
        out_host["ophist"] = nb.nvbt_opcode_hist(self.ctx)
        return self.hA.numel() * 4 + self.hB.numel() * 4, 8 * (4 + 3 * 18 + 3 + 66 + 2 * 16)

    def roofline(self, t_kernel_s, peaks):
        """Issue roofline ("alu") on the METHOD's own work: the minimal hook instructions of this rank's
        launch (BB-entry hooks at the K + 3 block instances, guard hooks at pc 7 and K x pc 15, divergence
        hooks at the 2K + 1 global LD/ST events per warp) ÷ the instrumented kernel time,
        against 148 SMs x 4 schedulers x 1 warp-instr/clk at the max SM clock. The SGEMM's own 12 + 6K
        instructions per warp are not the method's work and are excluded (reported beside it)."""
        K, W = self.K, self.rank_warps
        hooks = (K + 3) * HOOK_OPS["count"] + (K + 1) * HOOK_OPS["guard"] + (2 * K + 1) * HOOK_OPS["mem"]
        ops = W * hooks
        peak = N_SM * 4 * peaks.get("sm_max_mhz", 1965.0) * 1e6
        ach = ops / t_kernel_s
        t = load_traffic("k_sgemm<6>")
        return {"bound": "alu", "achieved": ach / 1e9, "peak": peak / 1e9, "unit": "Gwarp-inst/s",
                "frac": ach / peak, "traffic": t["traffic_bytes_per_launch"] if t else None,
                "traffic_unit": "DRAM bytes per launch (ncu, profiles/r2_traffic.json)",
                "algorithmic_hook_warp_inst_per_launch": ops,
                "with_app_instructions_frac": (ops + W * self.per_warp) / t_kernel_s / peak}


def run_c2(args, torch, nb, dr, rank, world, local, peaks, peaks_src):
    wl = SgemmBench(torch, nb, dr, rank, world)
    dev = torch.device("cuda", local)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    timed_steps(torch, wl.instr, args.warmup, flush)
    timed_steps(torch, wl.plain, args.warmup, flush)
    t_plain = timed_steps(torch, wl.plain, args.steps, flush)
    wl.reset()
    barrier(world)
    torch.cuda.synchronize()
    l0 = nb.nvbt_launch_count(wl.ctx)
    with ClockSampler(local) as clk:
        barrier(world)
        torch.cuda.synchronize()
        t_instr = timed_steps(torch, wl.instr, args.steps, flush)
        torch.cuda.synchronize()
        barrier(world)
    gpu_launches = nb.nvbt_launch_count(wl.ctx) - l0
    merge_ms = 0.0
    if world > 1:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        merge(dr, wl.ctx, world)
        e1.record()
        e1.synchronize()
        merge_ms = max_over_ranks(e0.elapsed_time(e1), world)
    # the timed steps' merged result: exactly K x the per-launch closed form (I-3)
    cnt = nb.nvbt_count(wl.ctx)
    _, tot, _, _ = nb.nvbt_mem_divergence(wl.ctx)
    K = args.steps
    ok = (int(cnt[2]) == wl.events * K and int(tot[0]) == 67_141_632 * K and
          int(tot[1]) == int(tot[2]) == 1_108_344_832 * K)
    tot_instr = max_over_ranks(sum(t_instr), world)
    tot_plain = max_over_ranks(sum(t_plain), world)
    t_kernel = max_over_ranks(statistics.median(t_instr), world)
    value = wl.events * K / tot_instr
    # e2e through the public API with host buffers
    out = {}
    for _ in range(2):
        wl.e2e_step(out)
    torch.cuda.synchronize()
    barrier(world)
    e2e_steps = max(3, min(args.steps, 10))
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        h2d, d2h = wl.e2e_step(out)
    torch.cuda.synchronize()
    e2e_t = max_over_ranks(time.perf_counter() - t0, world)
    line = {
        "metric": METRIC, "value": value, "unit": "events/s", "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": 1e3 * tot_instr / K, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.desc, "M": wl.M, "N": wl.N, "K": wl.K, "warp_events_per_launch": wl.events,
                   "tools": "BBCOUNT|MEMDIV", "l2": "flushed between steps (256 MiB write)",
                   "parallelism": (f"CTA-row partition of the launch over {world} GPUs (nvbt_set_partition), "
                                   "one int64 all-reduce merge") if world > 1 else "1 GPU"},
        "slowdown": tot_instr / tot_plain, "plain_ms_per_launch": 1e3 * max_over_ranks(statistics.median(t_plain), world),
        "instr_ms_per_launch": 1e3 * t_kernel,
        "counts_check": "ok" if ok else f"mismatch W_issued {int(cnt[2])} != {wl.events * K}",
        "roofline": wl.roofline(statistics.median(t_instr), peaks),
        "e2e": {"value": wl.events * e2e_steps / e2e_t, "unit": "events/s", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h},
        "gpu_launches": int(gpu_launches), "clocks": clk.summary(), "peaks_source": peaks_src,
        "merge_ms": merge_ms,
        "paper_context": ("the paper's opcode-histogram tool (this path's a3): 36.4x average, up to 112x slowdown "
                          "fully instrumented, 2.3x with kernel sampling; TITAN V (Volta), SpecAccel (P:L278-280)"),
    }
    line["roofline"]["peak_source"] = f"148 SMs x 4 issue/clk x sm_max_mhz ({peaks_src})"
    # the binding resource of this workload is the application's own L1 traffic (the naive row-fastest
    # SGEMM is L1-wavefront-bound uninstrumented); the hooks run inside that bound
    line["app_bound"] = {"resource": "L1TEX wavefronts of the uninstrumented SGEMM",
                         "instr_speed_vs_plain": statistics.median(t_plain) / statistics.median(t_instr),
                         "ncu": "profiles/r2_ncu_summary_c2.txt: l1tex 98.6 % (plain) / 94.9 % (instrumented), "
                                "issue-active 7.0 % / 85.0 %"}
    line["ncu_per_event"] = {"instrumented": load_counters("k_sgemm<6>"), "plain": load_counters("k_sgemm<0>"),
                             "source": "profiles/r2_ncu_counters.json (ncu --set full, tools/prof_step.py c2)"}
    return line, wl


def c2_cpu_baseline(wl, nb):
    """cpu_baseline leg: the C oracle (all host cores) over the WHOLE C2 launch (same buffers, so the same
    events), timed; plus its 1-thread rate on a 1 % slice; its result must equal the GPU's per launch."""
    from oracle import coracle as co, programs
    prog = programs.sgemm()
    T = co.host_threads()
    a, b, c = wl.A.data_ptr(), wl.B.data_ptr(), wl.C.data_ptr()
    co.sgemm(prog, 64, 64, 64, a, b, c, threads=T)          # load + build outside the timing
    t0 = time.perf_counter()
    r = co.sgemm(prog, wl.M, wl.N, wl.K, a, b, c, threads=T)
    dt = time.perf_counter() - t0
    sl = wl.nw // 100
    t1 = time.perf_counter()
    co.sgemm(prog, wl.M, wl.N, wl.K, a, b, c, warps=(0, sl), threads=1)
    dt1 = time.perf_counter() - t1
    cnt = nb.nvbt_count(wl.ctx).astype(np.int64)
    per, tot, hs, hl = nb.nvbt_mem_divergence(wl.ctx)
    steps = wl.launched
    match = (np.array_equal(cnt, steps * r["counts"]) and np.array_equal(per[:, 1].astype(np.int64), steps * r["mem_S"])
             and np.array_equal(per[:, 2].astype(np.int64), steps * r["mem_L"])
             and np.array_equal(hs.astype(np.int64), steps * r["hS"]))
    return {"value": wl.events / dt, "unit": "events/s", "cores": T, "kind": "oracle",
            "sample": f"the whole C2 launch ({wl.events} warp events), C oracle (oracle/c) on {T} threads",
            "cpu_model": cpu_model(), "one_thread_value": sl * wl.per_warp / dt1,
            "one_thread_sample": f"warps [0, {sl}) (1 %) on 1 thread", "matches_gpu": bool(match)}


# --------------------------------------------------------------------------- C1 vectorAdd
def run_c1(args, torch, nb, dr, rank, world, local, steps):
    """C1: vectorAdd N = 65536, instruction counts + opcode histogram. A launch moves 786 KB, so launch
    overhead dominates: launches are batched into one CUDA graph of `reps` launches (captured on the
    context's stream) and each replay is timed. Counts two ways, identical results (I-5): BBCOUNT (hooks at
    block leaders and guarded pcs) is the config's value, COUNT (a hook at every pc) beside it."""
    from synth import uniform_f32
    N, reps = 65536, 200
    s = torch.cuda.Stream()
    ctxs = {}
    for name in ("COUNT", "BBCOUNT"):
        ctxs[name] = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.OPHIST | nb.BB, stream=s)
        if world > 1:
            nb.nvbt_set_partition(ctxs[name], rank, world)
    a = torch.from_numpy(uniform_f32(N, 1)).cuda()
    b = torch.from_numpy(uniform_f32(N, 2)).cuda()
    c = torch.empty_like(a)
    torch.cuda.synchronize()

    def graph_of(ctx, tools):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                nb.nvbt_vectoradd(ctx, tools, a, b, c, N)
        return g

    graphs = {"plain": graph_of(ctxs["COUNT"], nb.TOOL_NONE), "COUNT": graph_of(ctxs["COUNT"], nb.TOOL_COUNT),
              "BBCOUNT": graph_of(ctxs["BBCOUNT"], nb.TOOL_BBCOUNT)}

    def timed(g, n):
        ts = []
        for _ in range(n):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(s):
                e0.record(s)
                g.replay()
                e1.record(s)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        return ts

    for g in graphs.values():
        timed(g, 3)
    t = {}
    for name in ("plain", "COUNT", "BBCOUNT"):
        if name != "plain":
            nb.nvbt_reset(ctxs[name])
        barrier(world)
        t[name] = max_over_ranks(sum(timed(graphs[name], steps)), world) / (steps * reps)
    res = {}
    for name in ("COUNT", "BBCOUNT"):
        merge(dr, ctxs[name], world)
        res[name] = (nb.nvbt_count(ctxs[name]), nb.nvbt_opcode_hist(ctxs[name]))
    same = (np.array_equal(res["COUNT"][0], res["BBCOUNT"][0]) and
            all(np.array_equal(x, y) for x, y in zip(res["COUNT"][1], res["BBCOUNT"][1])))
    ev = int(res["BBCOUNT"][0][2]) // (steps * reps)
    ok = ev == 26624 and int(res["BBCOUNT"][0][3]) == 24576 * steps * reps and same
    return {"value": 26624 / t["BBCOUNT"], "unit": "events/s", "steps": steps, "launches_per_step": reps,
            "workload": "C1 vectorAdd N=65536 (256 thr/CTA), counts + opcode histogram, tools BBCOUNT",
            "slowdown": t["BBCOUNT"] / t["plain"], "plain_us_per_launch": 1e6 * t["plain"],
            "instr_us_per_launch": 1e6 * t["BBCOUNT"],
            "per_instruction_hooks": {"tools": "COUNT", "value": 26624 / t["COUNT"], "slowdown": t["COUNT"] / t["plain"]},
            "counts_check": ("ok: W_issued 26,624 and W_exec 24,576 per launch (I-3), COUNT == BBCOUNT counts "
                             "and opcode histograms") if ok else f"mismatch: {ev} events per launch, same={same}",
            "roofline": {"bound": "launch", "note": "26,624 warp events per launch: launch latency, not a "
                         "throughput roofline (CUDA-graph replays)"}}


# --------------------------------------------------------------------------- C3 BFS
def run_c3(args, torch, nb, dr, rank, world, local, steps):
    """C3: BFS on the R-MAT scale-20 graph (edge factor 16) with BB-entry counting; a step is one whole
    BFS. N > 1: vertex-range partition with the per-level MAX exchanges (drivers.run_bfs_dist)."""
    from synth import rmat_csr, bfs_source
    rowptr, col = rmat_csr(args.bfs_scale, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    nw = nb.nvbt_workload_warps(nb.W_BFS, n)
    rp, cl = torch.from_numpy(rowptr).cuda(), torch.from_numpy(col).cuda()
    ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    if world > 1:
        nb.nvbt_set_partition(ctx, rank, world)
    bufs = dr.bfs_buffers(n, "cuda")
    if world > 1:
        bfs = lambda t: dr.run_bfs_dist(ctx, t, rp, cl, src, bufs)
    else:
        bfs = lambda t: dr.run_bfs(ctx, t, rp, cl, src, bufs)
    for _ in range(2):
        bfs(nb.TOOL_NONE)
        bfs(nb.TOOL_BBCOUNT)
    barrier(world)
    tp = max_over_ranks(sum(timed_steps(torch, lambda: bfs(nb.TOOL_NONE), steps)), world)
    nb.nvbt_reset(ctx)
    barrier(world)
    ti = max_over_ranks(sum(timed_steps(torch, lambda: bfs(nb.TOOL_BBCOUNT), steps)), world)
    _, levels = bfs(nb.TOOL_NONE)
    merge(dr, ctx, world)
    cnt = nb.nvbt_count(ctx)
    bb = nb.nvbt_bb_count(ctx)
    ev = int(cnt[2]) // steps
    # every kernel-1 launch is entered by every warp: Ent_w(block 0) = levels x warps per BFS
    ok = int(bb[0, 0]) == levels * nw * steps
    return {"value": ev * steps / ti, "unit": "events/s", "steps": steps,
            "workload": f"C3 BFS R-MAT scale {args.bfs_scale} ef16 (Graph500 a,b,c), tools BBCOUNT",
            "vertices": n, "directed_edges": int(len(col)), "levels": levels, "warp_events_per_bfs": ev,
            "slowdown": ti / tp, "plain_ms_per_bfs": 1e3 * tp / steps, "instr_ms_per_bfs": 1e3 * ti / steps,
            "counts_check": "ok: Ent_w(kernel 1 entry block) = levels x warps" if ok else
                            f"mismatch Ent_w {int(bb[0, 0])} != {levels * nw * steps}",
            "roofline": {"bound": "latency", "note": "the hub warp's serial edge loop (max degree ~6.5e4) "
                         "bounds both the plain and the instrumented BFS"}}


# --------------------------------------------------------------------------- C4 stencil + channel
def run_c4(args, torch, nb, dr, rank, world, local, steps, compact=False):
    """C4: 8192^2 5-point stencil x 100 iterations, every executed global LD/ST traced through the pinned
    host channel (288 B records, EM §5; with `compact` True / 128 the F3 transports of EM §5.1 / §5.2,
    decoded back to the same records on the host) and digested on the host; a step is the whole traced run. The
    drain runs on a host thread while the iterations are enqueued (N > 1: row slabs with P2P halos, one
    channel per rank). Device time from the first launch to the last kernel's end (the producers wait on
    the host ring, so it includes the transport), max over ranks."""
    from synth import uniform_f32
    n, iters = args.stencil_n, args.stencil_iters
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.TRACE)
    if world > 1:
        nb.nvbt_set_partition(ctx, rank, world)
    x0 = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
    buf0, buf1 = x0.clone(), torch.empty_like(x0)
    ring = torch.empty(nb.nvbt_channel_bytes(args.ring_records, compact=compact), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring, compact=compact)
    if world > 1:
        run = lambda t, it: dr.run_stencil_dist(ctx, t, buf0, buf1, n, it, rank, world, gather=False)
    else:
        run = lambda t, it: dr.run_stencil(ctx, t, buf0, buf1, n, it)

    def traced(it):
        d = nb.Digest()
        done = threading.Event()
        err = []

        def drain():   # the drain returns whenever the stream is idle with everything delivered
            try:
                while True:
                    fin = done.is_set()
                    nb.nvbt_channel_drain_digest(ch, timeout_us=900_000_000, digest=d)
                    if fin:
                        return
            except Exception as e:  # noqa: BLE001 - reported by the caller
                err.append(e)
        th = threading.Thread(target=drain)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record()
        th.start()
        run(nb.TOOL_TRACE, it)
        e1.record()
        done.set()
        th.join()
        torch.cuda.synchronize()
        if err:
            raise err[0]
        return e0.elapsed_time(e1) / 1e3, time.perf_counter() - t0, d.n_rec

    run(nb.TOOL_NONE, iters)
    tp = max_over_ranks(sum(timed_steps(torch, lambda: run(nb.TOOL_NONE, iters), max(steps, 3))), world) / max(steps, 3)
    traced(max(1, iters // 10))                                  # warm-up: 10 % of the iterations
    barrier(world)
    res = [traced(iters) for _ in range(steps)]
    dropped = nb.nvbt_channel_dropped(ch)
    t_dev = max_over_ranks(sum(r[0] for r in res), world) / steps
    t_wall = max_over_ranks(sum(r[1] for r in res), world) / steps
    recs = sum_over_ranks(res[-1][2], world)
    G = n // 32
    expect = iters * (4 * G + 6 * G * (n - 2))                   # SURVEY I-3 closed form
    dropped_all = sum_over_ranks(dropped, world)
    ok = int(recs) == expect and dropped_all == 0
    slot = nb.nvbt_channel_slot_bytes(compact)                     # ring stride per transport slot
    gbs = recs * (slot + 4) / t_dev / 1e9 / world                  # slots + commit tags per GPU link
    peak = d2h_peak()
    nb.nvbt_channel_close(ch)
    del ring
    transport = {False: "288 B records", True: "176 B compact slots (EM 5.1)", 128: "128 B line slots (EM 5.2)"}[compact]
    return {"value": recs / t_dev if ok else None, "unit": "records/s", "steps": steps,
            "workload": f"C4 stencil {n}^2 x {iters}, tools TRACE, {transport} to pinned host, digest drain",
            "records_per_s_measured": recs / t_dev, "transport_slot_bytes": slot,
            "records_per_run": int(recs), "records_expected": expect, "dropped": int(dropped_all),
            "slowdown": t_dev / tp, "plain_ms": 1e3 * tp, "traced_s": t_dev, "traced_wall_s": t_wall,
            "ring_slots": args.ring_records,
            "counts_check": "ok: records = iters x (4G + 6G(n-2)) (I-3), none dropped" if ok else
                            f"mismatch: {int(recs)} records, expected {expect}, dropped {int(dropped_all)}",
            "roofline": {"bound": "pcie", "achieved": gbs, "peak": peak, "unit": "GB/s", "frac": gbs / peak,
                         "peak_source": "measured SM-store D2H into pinned memory (profiles/r1_box_peaks.json)",
                         "algorithmic_bytes_per_record": slot + 4}}


# --------------------------------------------------------------------------- C5 replay
def _replay_traffic(chunk):
    """ncu DRAM bytes of one staged replay call on `chunk` events (captured at 2^26 events, scaled)."""
    tr = [load_traffic(k) for k in ("k_rpA<0>", "k_rpB")]
    if any(t is None for t in tr):
        return None
    return sum(t["traffic_bytes_per_launch"] for t in tr) / 67108864 * chunk


def run_c5(args, torch, nb, dr, rank, world, local, steps, peaks, peaks_src):
    """C5: staged replay (counts, histograms, divergence) of 10^10 generated events in 2^27-event chunks;
    generation is not timed; N > 1: contiguous event-index ranges per rank. Inputs (36.5 GB per chunk)
    exceed L2."""
    n_total, chunk = args.replay_events, 1 << 27
    lo, hi = dr.shard_range(n_total, rank, world)
    n = hi - lo
    ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)
    hdr = torch.empty(chunk * 16, dtype=torch.uint8, device="cuda")
    addr = torch.empty(chunk * 256, dtype=torch.uint8, device="cuda")
    scratch = torch.empty(nb.nvbt_replay_scratch_size(ctx, chunk), dtype=torch.uint8, device="cuda")
    for _ in range(2):
        nb.nvbt_gen_events(ctx, SEED, lo, min(chunk, n), hdr, addr)
        nb.nvbt_replay_staged(ctx, hdr, addr, min(chunk, n), scratch)
    nb.nvbt_reset(ctx)
    torch.cuda.synchronize()
    barrier(world)

    gen_t = [0.0]

    def step():
        t = 0.0
        off = 0
        while off < n:
            m = min(chunk, n - off)
            g0, e0, e1 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            g0.record()
            nb.nvbt_gen_events(ctx, SEED, lo + off, m, hdr, addr)
            e0.record()
            nb.nvbt_replay_staged(ctx, hdr, addr, m, scratch)
            e1.record()
            e1.synchronize()
            t += e0.elapsed_time(e1) / 1e3
            gen_t[0] += g0.elapsed_time(e0) / 1e3
            off += m
        return t

    ts = [step() for _ in range(steps)]
    t_gen = max_over_ranks(gen_t[0] / steps, world)
    _, tot, _, _ = nb.nvbt_mem_divergence(ctx)
    mem_exec = int(tot[0]) // steps
    t_rank = sum(ts) / steps
    ach = (16 * n + 256 * mem_exec) / t_rank / 1e9
    merge(dr, ctx, world)
    cnt = nb.nvbt_count(ctx)
    t_all = max_over_ranks(t_rank, world)
    ok = int(cnt[2]) == steps * n_total
    del hdr, addr, scratch
    torch.cuda.empty_cache()
    return {"value": n_total / t_all, "unit": "events/s", "steps": steps,
            "workload": f"C5 staged trace replay of {n_total:.3g} generated events (counts, histograms, divergence)",
            "ms_per_step": 1e3 * t_all, "chunk": chunk,
            "generation_ms_per_step": 1e3 * t_gen,
            "generate_and_replay_events_per_s": n_total / (t_all + t_gen),
            "counts_check": "ok: W_issued = events" if ok else f"mismatch W_issued {int(cnt[2])}",
            "roofline": {"bound": "hbm", "achieved": ach, "peak": float(peaks["hbm_gbs"]), "unit": "GB/s",
                         "frac": ach / float(peaks["hbm_gbs"]), "peak_source": peaks_src,
                         "algorithmic_bytes": "16 per header + 256 per executed memory event (per rank)",
                         "traffic": _replay_traffic(chunk),
                         "traffic_unit": "DRAM bytes per 2^27-event call (ncu at 2^26, scaled)",
                         "kernel": "nvbt_replay_staged = k_rpA (headers, list) + k_rpB (slots)"}}


# --------------------------------------------------------------------------- NEXT-row profiling lines (F1, F2, F4)
def run_f2(args, torch, nb, dr, local):
    """F2: C4's traced stencil (8192^2, --f2-iters iterations) with the trace kept in an HBM ring and
    analysed on the GPU (per-launch footprint) instead of drained to the host. A step = traced run
    + consumer kernel; the ring is re-zeroed between steps outside the timed region."""
    from synth import uniform_f32
    peaks, peaks_src = load_peaks()
    n, iters = args.stencil_n, args.f2_iters
    G = n // 32
    per_iter = 2 * (n * n // 32) + 4 * (n - 2) * G
    cap = per_iter * iters
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.TRACE)
    x0 = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
    buf0, buf1 = x0.clone(), torch.empty_like(x0)
    slack = cap // 50 + torch.cuda.get_device_properties(0).multi_processor_count * 4096   # nvbt.h sizing
    ring = torch.empty(64 + 288 * (cap + slack), dtype=torch.uint8, device="cuda")
    regions = iters * 2 * (-(-n * n * 4 // (1 << 20)) + 1)          # (launch, 1 MB region) pairs
    slots = 1 << (2 * regions - 1).bit_length()
    scratch = torch.empty(513 * slots + 3 * iters + 1, dtype=torch.int64, device="cuda")
    for _ in range(args.warmup):
        dr.run_stencil(ctx, nb.TOOL_NONE, buf0, buf1, n, iters)
    tp = _timed_events(torch, lambda: dr.run_stencil(ctx, nb.TOOL_NONE, buf0, buf1, n, iters), args.steps)
    res, kern, fp = [], [], None
    l0 = nb.nvbt_launch_count(ctx)
    with ClockSampler(local) as clk:
        for step in range(args.warmup + args.steps):
            ch = nb.nvbt_channel_open(ctx, ring)
            nb.nvbt_reset(ctx)                               # launch ids restart at 0
            torch.cuda.synchronize()
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record()
            dr.run_stencil(ctx, nb.TOOL_TRACE, buf0, buf1, n, iters)
            e1.record()
            tk = []
            fp = nb.nvbt_trace_footprint(ch, iters, table_slots=slots, scratch=scratch, timing=tk)
            e2.record()
            e2.synchronize()
            dropped = nb.nvbt_channel_dropped(ch)
            nb.nvbt_channel_close(ch)
            if step >= args.warmup:
                res.append((e0.elapsed_time(e1) / 1e3, e1.elapsed_time(e2) / 1e3))
                kern.append(tk[0])
    launches = nb.nvbt_launch_count(ctx) - l0
    recs = int(fp[:, 2].sum())
    t_tr = sum(r[0] for r in res) / len(res)
    t_fp = sum(r[1] for r in res) / len(res)
    t_k = sum(kern) / len(kern)
    ach = recs * 288 / t_k / 1e9
    exp_s, exp_l = 2 * n * n * 4 // 32, 2 * n * n * 4 // 128    # in + out grids, whole sectors / lines
    return {"metric": "traced warp-level memory events analysed on GPU per second (F2)",
            "value": recs / (t_tr + t_fp), "unit": "records/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * (t_tr + t_fp), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"F2 stencil {n}^2 x {iters}, tools TRACE, HBM ring + GPU footprint consumer",
                       "ring_GB": ring.numel() / 1e9, "table_slots": slots,
                       "l2": "records (36 GB) larger than L2"},
            "records_per_run": recs, "records_expected": cap, "dropped": dropped,
            "trace_ms": 1e3 * t_tr, "consumer_ms": 1e3 * t_fp, "consumer_kernel_ms": 1e3 * t_k,
            "plain_ms": 1e3 * sum(tp) / len(tp), "slowdown_trace_only": t_tr / (sum(tp) / len(tp)),
            "footprint_launch0": [int(x) for x in fp[0]], "footprint_expected": [exp_s, exp_l],
            "roofline": {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                         "frac": ach / peaks["hbm_gbs"], "peak_source": peaks_src, "kernel": "k_footprint",
                         "algorithmic_bytes_per_launch": recs * 288,
                         "traffic": (load_traffic("k_footprint") or {}).get("traffic_bytes_per_record", 0) * recs or None,
                         "traffic_unit": "DRAM bytes per consumer launch (ncu per-record figure at 4096^2 x 4, scaled)"},
            "gpu_launches": int(launches) // (args.warmup + args.steps), "clocks": clk.summary()}


def run_f1(args, torch, nb, dr, local):
    """F1 kernel sampling on C4's stencil (8192^2 x 100, BBCOUNT|MEMDIV): plain vs every launch
    instrumented vs one instrumented launch per grid shape."""
    from synth import uniform_f32
    n, iters = args.stencil_n, args.stencil_iters
    flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV
    full, samp, scratch = (nb.nvbt_init(nb.W_STENCIL, flags) for _ in range(3))
    x0 = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
    b = (x0.clone(), torch.empty_like(x0))
    tools = nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV

    def run(mode):
        sampler = dr.KernelSampler(samp, scratch) if mode == "sampled" else None
        if mode == "sampled":
            nb.nvbt_reset(samp)
        for it in range(iters):
            src, dst = b[it % 2], b[(it + 1) % 2]
            if mode == "plain":
                nb.nvbt_stencil(full, nb.TOOL_NONE, src, dst, n)
            elif mode == "full":
                nb.nvbt_stencil(full, tools, src, dst, n)
            else:
                sampler.launch(("stencil", n), lambda c, t: nb.nvbt_stencil(c, t, src, dst, n), tools)
        if sampler:
            sampler.finish()

    res = {}
    exact = None
    for mode in ("plain", "full", "sampled"):
        for _ in range(args.warmup):
            run(mode)
        nb.nvbt_reset(full)
        res[mode] = _timed_events(torch, lambda: run(mode), args.steps)
        if mode == "full":
            exact = nb.nvbt_count(full).astype("int64") // args.steps
    est = nb.nvbt_count(samp).astype("int64")
    err = float(abs(est[2] - exact[2])) / float(exact[2])
    tp, tf, ts = (sum(res[m]) / len(res[m]) for m in ("plain", "full", "sampled"))
    return {"metric": "kernel-sampling slowdown vs uninstrumented (F1)", "value": ts / tp, "unit": "x",
            "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * ts,
            "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"F1 sampling on C4 stencil {n}^2 x {iters}, tools BBCOUNT|MEMDIV"},
            "full_slowdown": tf / tp, "sampled_slowdown": ts / tp, "warp_issued_rel_error": err,
            "paper_context": "36.4x full vs 2.3x sampled on TITAN V / SpecAccel (P:L280)"}


def run_f4(args, torch, nb, dr, local):
    """F4 instruction emulation (EM §3.6): n_fft warp-wide 32-point FFTs, the kernel using the
    proxy WFFT32 with the emulation tool vs the same transform written in CUDA, each plain and instrumented.
    Inputs and outputs (2 x n_fft x 256 B) exceed L2, so no flush is needed between steps."""
    n_fft, ctas = args.fft_n, args.fft_ctas
    peaks, peaks_src = load_peaks()
    g = torch.Generator(device="cuda").manual_seed(9)
    x = (torch.rand((n_fft, 32, 2), generator=g, device="cuda") * 2 - 1).view(torch.complex64).reshape(n_fft, 32)
    X = torch.empty_like(x)
    flags = nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV
    cemu, csw = nb.nvbt_init(nb.W_WFFT_EMU, flags), nb.nvbt_init(nb.W_WFFT_SW, flags)
    P, S = nb.WFFT_PROXY, nb.WFFT_SOFTWARE
    modes = {
        "proxy_plain": (cemu, P, nb.TOOL_NONE),   # native proxy = register move: a pure copy (memory bound)
        "sw_plain": (csw, S, nb.TOOL_NONE), "emu_only": (cemu, P, nb.TOOL_EMU),
        "sw_bbcount_memdiv": (csw, S, nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV),
        "emu_bbcount_memdiv": (cemu, P, nb.TOOL_EMU | nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV),
        "sw_count": (csw, S, nb.TOOL_COUNT), "emu_count": (cemu, P, nb.TOOL_EMU | nb.TOOL_COUNT),
    }
    res, warp_inst, grids = {}, {}, {}
    for name, (ctx, v, t) in modes.items():
        g_ctas = ctas if ctas > 0 else nb.nvbt_wfft32_max_ctas(t, v, local)   # one resident wave
        grids[name] = g_ctas
        f = lambda: nb.nvbt_wfft32(ctx, t, v, x, X, n_fft, g_ctas)
        _timed_events(torch, f, args.warmup)
        nb.nvbt_reset(ctx)
        if name == "emu_count":
            with ClockSampler(local) as clk:
                res[name] = _timed_events(torch, f, args.steps)
        else:
            res[name] = _timed_events(torch, f, args.steps)
        if t & (nb.TOOL_COUNT | nb.TOOL_BBCOUNT):
            warp_inst[name] = int(nb.nvbt_count(ctx)[2]) // args.steps
    med = {k: statistics.median(v) for k, v in res.items()}
    head = "emu_count"          # the paper's combination: emulation + the instruction-count tool
    ev_launch = warp_inst[head]
    t_k = med[head]
    bytes_launch = 512 * n_fft                       # algorithmic: read x, write X once
    hbm_peak = float(peaks["hbm_gbs"])
    body = {k: warp_inst[k] / n_fft for k in warp_inst}   # per transform (incl. the per-warp prologue share)
    return {"metric": METRIC, "value": ev_launch * args.steps / sum(res[head]), "unit": "events/s", "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(res[head]) / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"F4 WFFT32 emulation: {n_fft} warp-wide 32-point FFTs, persistent grid "
                                   "(one resident wave), tools EMU|COUNT", "n_fft": n_fft, "ctas": grids,
                       "l2": "inputs+outputs 2 x n_fft x 256 B > L2, no flush"},
            "fft_per_s": {k: n_fft / v for k, v in med.items()},
            "ms_per_launch": {k: 1e3 * v for k, v in med.items()},
            "slowdown_vs_sw_plain": {k: v / med["sw_plain"] for k, v in med.items()},
            "warp_instr_per_launch": warp_inst,
            "warp_instr_per_fft_approx": body,
            "roofline": {"bound": "hbm", "achieved": bytes_launch / t_k / 1e9, "peak": hbm_peak, "unit": "GB/s",
                         "frac": bytes_launch / t_k / 1e9 / hbm_peak,
                         "traffic": (load_traffic("k_wfft<17,0>") or {}).get("traffic_bytes_per_launch"),
                         "traffic_unit": "DRAM bytes per launch (ncu, profiles/r2_traffic.json)",
                         "algorithmic_bytes_per_launch": bytes_launch, "kernel": "k_wfft<EMU|COUNT, proxy>"},
            "sw_plain_hbm_frac": bytes_launch / med["sw_plain"] / 1e9 / hbm_peak,
            "clocks": clk.summary(), "peaks_source": peaks_src,
            "paper_context": "21 vs 150 instructions per warp with and without WFFT32 (P:L295), parity-unpinned"}


# --------------------------------------------------------------------------- main
def run_ours(args):
    import torch
    rank, world, local = dist_setup(args)
    import paper_conf_micro_villasnk19_b200 as pkg
    nb, dr = pkg.nvbt, pkg.drivers
    peaks, peaks_src = load_peaks()
    if args.workload in ("f1", "f2", "f4"):
        line = {"f1": run_f1, "f2": run_f2, "f4": run_f4}[args.workload](args, torch, nb, dr, local)
        if rank == 0:
            print(json.dumps(line), flush=True)
        return
    line, wl = run_c2(args, torch, nb, dr, rank, world, local, peaks, peaks_src)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = c2_cpu_baseline(wl, nb)
    del wl
    torch.cuda.empty_cache()
    wanted = [c for c in args.configs.split(",") if c and c != "none"]
    cfg = {}
    for c in wanted:
        torch.cuda.nvtx.range_push(f"nvbt bench {c}")
        if c == "c1":
            cfg["c1"] = run_c1(args, torch, nb, dr, rank, world, local, args.steps)
        elif c == "c3":
            cfg["c3"] = run_c3(args, torch, nb, dr, rank, world, local, min(args.steps, 5))
        elif c == "c4":
            cfg["c4"] = run_c4(args, torch, nb, dr, rank, world, local, args.c4_steps)
        elif c == "c4_compact":
            cfg["c4_compact"] = run_c4(args, torch, nb, dr, rank, world, local, args.c4_steps, compact=True)
        elif c == "c4_line":
            cfg["c4_line"] = run_c4(args, torch, nb, dr, rank, world, local, args.c4_steps, compact=128)
        elif c == "c5":
            cfg["c5"] = run_c5(args, torch, nb, dr, rank, world, local, args.c5_steps, peaks, peaks_src)
        torch.cuda.nvtx.range_pop()
        torch.cuda.empty_cache()
    if cfg:
        line["configs"] = cfg
    if world > 1:
        line["allreduce_latency"] = allreduce_latency(world)
        if HOST_PLACEMENT is not None:
            line["host_placement_rank0"] = HOST_PLACEMENT
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


def run_reference(args):
    """Reference arm = the CPU oracle (this tier has no runnable reference): the C oracle
    (oracle/c, multithreaded, plain event-by-event EM §2) on all host cores; one step = one whole C2 launch
    (the same 201,719,808 warp events the GPU step instruments)."""
    if int(os.environ.get("RANK", "0")) != 0:
        return
    from oracle import coracle as co, programs
    prog = programs.sgemm()
    M = N = K = 1024
    T = co.host_threads()
    events = (M // 32) * (N // 8) * 8 * (12 + 6 * K)
    base = 1 << 32
    ptrs = (base, base + (8 << 20), base + (16 << 20))
    for _ in range(args.warmup):
        co.sgemm(prog, M, N, K, *ptrs, threads=T, warps=(0, 3276))
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        co.sgemm(prog, M, N, K, *ptrs, threads=T)
        ts.append(time.perf_counter() - t0)
    value = events * args.steps / sum(ts)
    sample = f"the whole C2 launch ({events} warp events) per step, C oracle on {T} threads"
    line = {
        "metric": METRIC, "value": value, "unit": "events/s", "n_gpus": int(os.environ.get("WORLD_SIZE", args.gpus)),
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(ts) / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": SgemmBench.desc, "M": M, "N": N, "K": K}, "impl": "reference",
        "cpu_baseline": {"value": value, "unit": "events/s", "cores": T, "kind": "oracle", "sample": sample,
                         "cpu_model": cpu_model()},
        "e2e": {"value": value, "unit": "events/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=["c2", "f1", "f2", "f4"], default="c2",
                    help="c2: the headline line with --configs beside it; f1/f2/f4: NEXT-row profiling lines")
    ap.add_argument("--configs", default="c1,c3,c4,c4_compact,c4_line,c5", help="configs measured beside C2 ('none' for C2 only)")
    ap.add_argument("--c4-steps", type=int, default=2)
    ap.add_argument("--c5-steps", type=int, default=3)
    ap.add_argument("--fft-n", type=int, default=1 << 24, help="F4: transforms per launch")
    ap.add_argument("--fft-ctas", type=int, default=0, help="F4: grid (0 = one resident wave per kernel)")
    ap.add_argument("--f2-iters", type=int, default=10, help="F2: stencil iterations kept in the HBM ring")
    ap.add_argument("--bfs-scale", type=int, default=20)
    ap.add_argument("--stencil-n", type=int, default=8192)
    ap.add_argument("--stencil-iters", type=int, default=100)
    ap.add_argument("--ring-records", type=int, default=1 << 22)
    ap.add_argument("--replay-events", type=int, default=10**10)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    elif args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args.gpus))
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
