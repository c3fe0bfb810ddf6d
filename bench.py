#!/usr/bin/env python
"""nvbt benchmark: instrumented warp-instruction events/s and slowdown vs the uninstrumented kernel.

Default workload (BASELINE.json configs[1]): C2 — naive row-fastest SGEMM 1024^3 with the full tool set
compiled in (counts, opcode/BB histograms, per-instruction memory divergence), one step = one
instrumented launch; with N > 1 each rank runs its own instance and the counters are merged once by an
int64 all-reduce after the timed steps. Other workloads
(`--workload c1|c3|c4|c5`) are for profiling; the driver's bench line is C2.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c2] [--impl ours|reference]

Multi-GPU (weak scaling): torchrun, one rank per GPU, every rank runs its own instance; the time of
the job is the max over ranks. Timing: CUDA events on the context's stream around each step, L2
flushed (256 MiB write) between steps, clocks sampled with nvidia-smi during the timed region.
"""
from __future__ import annotations

import argparse
import json
import os
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


def load_traffic(kernel):
    """DRAM bytes per launch of `kernel` from the committed ncu capture (profiles/r1_traffic.json)."""
    try:
        with open(os.path.join(ROOT, "profiles", "r1_traffic.json")) as f:
            return json.load(f).get(kernel)
    except Exception:
        return None


def load_counters(kernel, keys=("warp_inst_per_unit", "dram_bytes_per_unit", "shared_atomic_wavefronts_per_unit",
                                 "global_atomic_sectors_per_unit", "issue_active_pct")):
    """ncu counters per unit of work of `kernel` from the committed capture (profiles/r1_ncu_counters.json)."""
    try:
        with open(os.path.join(ROOT, "profiles", "r1_ncu_counters.json")) as f:
            d = json.load(f).get(kernel)
    except Exception:
        return None
    return None if d is None else {k: d[k] for k in keys if k in d}


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return p, "measured"
    except Exception:
        return PEAKS_FALLBACK, "fallback"


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
def dist_setup(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("NVBT_BENCH_SAME_GPU"):   # test hook: all ranks on GPU 0 (with a gloo backend)
        local = 0
    if args.impl == "ours":
        torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        backend = os.environ.get("NVBT_BENCH_BACKEND", "nccl" if args.impl == "ours" else "gloo")
        kw = {"device_id": torch.device("cuda", local)} if backend == "nccl" else {}
        dist.init_process_group(backend, **kw)
    return rank, world, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(x, world, device=None):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x, world, device=None):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


# --------------------------------------------------------------------------- C2 SGEMM
class SgemmBench:
    name = "c2"
    M = N = K = 1024
    desc = "C2 naive row-fastest SGEMM 1024^3 (fp32), tools BBCOUNT|MEMDIV (counts, opcode+BB histograms via BB-entry hooks, divergence)"

    def __init__(self, torch, nb, dr, world):
        self.torch, self.nb, self.dr, self.world = torch, nb, dr, world
        from synth import uniform_f32
        M, N, K = self.M, self.N, self.K
        self.nw = nb.nvbt_workload_warps(nb.W_SGEMM, M, N)
        self.ctx = nb.nvbt_init(nb.W_SGEMM, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)
        self.tools = nb.TOOL_BBCOUNT | nb.TOOL_MEMDIV
        self.hA = torch.from_numpy(uniform_f32((M, K), 3, -1, 1)).pin_memory()
        self.hB = torch.from_numpy(uniform_f32((K, N), 4, -1, 1)).pin_memory()
        self.A, self.B = self.hA.cuda(), self.hB.cuda()
        self.C = torch.empty(M, N, device="cuda")
        # events per launch (EM §3.2): every warp runs 12 + 6K warp-level instructions
        self.events = self.nw * (12 + 6 * K)
        self.kernels_per_step = 1

    def plain(self):
        self.nb.nvbt_sgemm(self.ctx, self.nb.TOOL_NONE, self.A, self.B, self.C, self.M, self.N, self.K)

    def instr(self):
        self.nb.nvbt_sgemm(self.ctx, self.tools, self.A, self.B, self.C, self.M, self.N, self.K)

    def e2e_step(self, out_host):
        """Through the public API with host buffers: H2D inputs, instrumented launch, read results."""
        nb = self.nb
        self.A.copy_(self.hA, non_blocking=True)
        self.B.copy_(self.hB, non_blocking=True)
        nb.nvbt_sgemm(self.ctx, self.tools, self.A, self.B, self.C, self.M, self.N, self.K)
        out_host["counts"] = nb.nvbt_count(self.ctx)
        out_host["memdiv"] = nb.nvbt_mem_divergence(self.ctx)
        out_host["ophist"] = nb.nvbt_opcode_hist(self.ctx)
        return self.hA.numel() * 4 + self.hB.numel() * 4, 8 * (4 + 3 * 18 + 3 + 66 + 2 * 16)

    def roofline(self, t_kernel_s, peaks):
        """Issue roofline ("alu"): algorithmic warp-instructions per launch ÷ launch time vs
        148 SMs x 4 schedulers x 1 warp-instr/clk at the max SM clock."""
        K, W = self.K, self.nw
        # app instructions (one per warp-level event) + BB-entry hooks at the 3 + K leaders + guard
        # hooks at pc7 and K x pc15 + divergence hooks at the 2K + 1 global LD/ST events
        per_warp = (12 + 6 * K) + (K + 3) * HOOK_OPS["count"] + (K + 1) * HOOK_OPS["guard"] + \
            (2 * K + 1) * HOOK_OPS["mem"]
        ops = W * per_warp
        peak = N_SM * 4 * peaks.get("sm_max_mhz", 1965.0) * 1e6
        ach = ops / t_kernel_s
        t = load_traffic("k_sgemm<6>")
        return {"bound": "alu", "achieved": ach / 1e9, "peak": peak / 1e9, "unit": "Gwarp-inst/s",
                "frac": ach / peak, "traffic": t["traffic_bytes_per_launch"] if t else None,
                "traffic_unit": "DRAM bytes per launch (ncu, profiles/r1_traffic.json)",
                "algorithmic_warp_inst_per_launch": ops}

    def oracle_sample(self, budget_s):
        """The oracle on a bounded sample of the same workload: whole warps, full K."""
        from oracle import events as ev, programs
        from oracle.models import sgemm as m_sg
        acc = ev.Accumulator(programs.sgemm())
        rng = np.random.default_rng(1)
        warps = np.sort(rng.choice(self.nw, size=64, replace=False))
        t0 = time.perf_counter()
        done = 0
        while True:
            m_sg.run(acc, self.M, self.N, self.K, self.A.data_ptr(), self.B.data_ptr(), self.C.data_ptr(),
                     warps=warps)
            done += len(warps) * (12 + 6 * self.K)
            if time.perf_counter() - t0 > budget_s:
                break
        dt = time.perf_counter() - t0
        return done / dt, f"{done} warp events: SGEMM 1024^3 oracle model on 64 sampled warps x full K"


# hook instruction costs per event used for the issue roofline (minimal SASS per hook)
HOOK_OPS = {"count": 4, "guard": 6, "mem": 23}


# --------------------------------------------------------------------------- C5 replay
class ReplayBench:
    name = "c5"
    desc = "C5 trace replay of 10^10 generated events (counts, histograms, divergence), 2^27-event chunks"

    def __init__(self, torch, nb, dr, world, rank, n_total=10**10, chunk=1 << 27, staged=True):
        self.torch, self.nb, self.dr = torch, nb, dr
        self.lo, self.hi = dr.shard_range(n_total, rank, world)
        self.n = self.hi - self.lo
        self.chunk = chunk
        self.ctx = nb.nvbt_init(nb.W_REPLAY, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV)
        self.hdr = torch.empty(chunk * 16, dtype=torch.uint8, device="cuda")
        self.addr = torch.empty(chunk * 256, dtype=torch.uint8, device="cuda")
        # staged replay (two passes): the executed-memory-event list of one chunk (12 B per entry)
        self.scratch = torch.empty(nb.nvbt_replay_scratch_size(self.ctx, chunk), dtype=torch.uint8,
                                   device="cuda") if staged else None
        self.events = self.n
        self.kernels_per_step = -(-self.n // chunk)

    def oracle_sample(self, budget_s):
        """The oracle (generator + per-event definitions) on a bounded sample of the same event stream:
        consecutive 2^16-event chunks from the rank's first event until the budget is spent."""
        from oracle import events as ev, gen, programs
        acc = ev.Accumulator(programs.replay())
        t0 = time.perf_counter()
        done = 0
        while time.perf_counter() - t0 < budget_s:
            gen.replay(acc, self.lo + done, 1 << 16)
            done += 1 << 16
        dt = time.perf_counter() - t0
        return done / dt, f"{done} generated events from event {self.lo} (oracle replay incl. generation, 1 core)"

    def replay(self, m):
        if self.scratch is None:
            self.nb.nvbt_replay(self.ctx, self.hdr, self.addr, m)
        else:
            self.nb.nvbt_replay_staged(self.ctx, self.hdr, self.addr, m, self.scratch)

    def run(self, stream_events):
        """One step: generate (untimed) and replay (timed with events) every chunk."""
        torch, nb = self.torch, self.nb
        t = 0.0
        off = 0
        while off < self.n:
            m = min(self.chunk, self.n - off)
            nb.nvbt_gen_events(self.ctx, 0x4E5642544E564254, self.lo + off, m, self.hdr, self.addr)
            e0, e1 = stream_events
            e0.record()
            self.replay(m)
            e1.record()
            e1.synchronize()
            t += e0.elapsed_time(e1) / 1e3
            off += m
        return t


# --------------------------------------------------------------------------- main
def run_ours(args):
    import torch
    rank, world, local = dist_setup(args)
    import paper_conf_micro_villasnk19_b200 as pkg
    nb, dr = pkg.nvbt, pkg.drivers
    peaks, peaks_src = load_peaks()
    dev = torch.device("cuda", local)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    if args.workload == "c5":
        return run_replay(args, torch, nb, dr, rank, world, local, peaks, peaks_src)
    if args.workload in ("c1", "c3", "c4", "f1", "f2", "f4"):
        line = {"c1": run_c1, "c3": run_c3, "c4": run_c4, "f1": run_f1, "f2": run_f2, "f4": run_f4}[args.workload](
            args, torch, nb, dr, local)
        if rank == 0:
            print(json.dumps(line), flush=True)
        return

    wl = SgemmBench(torch, nb, dr, world)
    launches0 = nb.nvbt_launch_count(wl.ctx)

    def timed(fn, n):
        ts = []
        for _ in range(n):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) / 1e3)
        return ts

    # warm-up (untimed), plain baseline
    timed(wl.instr, args.warmup)
    timed(wl.plain, max(args.warmup, 3))
    t_plain = timed(wl.plain, args.steps)
    nb.nvbt_reset(wl.ctx)
    barrier(world)
    torch.cuda.synchronize()
    l0 = nb.nvbt_launch_count(wl.ctx)
    with ClockSampler(local) as clk:
        barrier(world)
        torch.cuda.synchronize()
        t_instr = timed(wl.instr, args.steps)
        torch.cuda.synchronize()
        barrier(world)
    gpu_launches = nb.nvbt_launch_count(wl.ctx) - l0
    # a8 merge: the per-GPU accumulators are summed once, by one int64 all-reduce (EM §4)
    merge_ms = 0.0
    if world > 1:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        dr.merge(wl.ctx)
        e1.record()
        e1.synchronize()
        merge_ms = e0.elapsed_time(e1)
    # result check of the timed steps: exactly K x the per-launch closed form (I-3)
    cnt = nb.nvbt_count(wl.ctx)
    expect = wl.events * args.steps * (world if world > 1 else 1)
    ok = int(cnt[2]) == expect
    tot_instr = max_over_ranks(sum(t_instr), world, dev)
    tot_plain = max_over_ranks(sum(t_plain), world, dev)
    events_all = wl.events * args.steps * world
    value = events_all / tot_instr
    slowdown = tot_instr / tot_plain
    t_kernel = statistics.median(t_instr)
    # e2e through the public API with host buffers
    out = {}
    for _ in range(2):
        wl.e2e_step(out)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    e2e_steps = max(3, min(args.steps, 10))
    for _ in range(e2e_steps):
        h2d, d2h = wl.e2e_step(out)
    torch.cuda.synchronize()
    e2e_t = max_over_ranks(time.perf_counter() - t0, world, dev)
    e2e_value = wl.events * e2e_steps * world / e2e_t
    line = {
        "metric": METRIC, "value": value, "unit": "events/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * tot_instr / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.desc, "M": wl.M, "N": wl.N, "K": wl.K, "warp_events_per_launch": wl.events,
                   "tools": "BBCOUNT|MEMDIV", "l2": "flushed between steps (256 MiB write)",
                   "parallelism": f"replicas x{world}, one int64 all-reduce merge of the counters" if world > 1 else "1 GPU"},
        "slowdown": slowdown, "plain_ms_per_launch": 1e3 * statistics.median(t_plain),
        "instr_ms_per_launch": 1e3 * t_kernel, "counts_check": "ok" if ok else f"mismatch {int(cnt[2])} != {expect}",
        "roofline": wl.roofline(t_kernel, peaks),
        "e2e": {"value": e2e_value, "unit": "events/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h},
        "gpu_launches": int(gpu_launches), "clocks": clk.summary(), "peaks_source": peaks_src,
        "merge_ms": merge_ms,
    }
    line["roofline"]["peak_source"] = f"148 SMs x 4 issue/clk x sm_max_mhz ({peaks_src})"
    # the binding resource of this workload is the application's own L1 traffic (the naive row-fastest
    # SGEMM is L1-wavefront-bound uninstrumented); the hooks run inside that bound
    line["app_bound"] = {"resource": "L1TEX wavefronts of the uninstrumented SGEMM",
                         "instr_speed_vs_plain": statistics.median(t_plain) / t_kernel,
                         "ncu": "profiles/r1_ncu_summary_c2_c5.txt: l1tex 98.8 % (plain) / 95.2 % (instrumented), "
                                "issue-active 6.9 % / 85.2 %"}
    # ncu evidence per warp event (the north_star's instructions per event and atomic traffic)
    line["ncu_per_event"] = {"instrumented": load_counters("k_sgemm<6>"), "plain": load_counters("k_sgemm<0>"),
                             "source": "profiles/r1_ncu_counters.json (ncu --set full, tools/prof_step.py c2)"}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, sample = wl.oracle_sample(args.cpu_budget)
        line["cpu_baseline"] = {"value": rate, "unit": "events/s", "cores": 1, "kind": "oracle", "sample": sample}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


def _replay_traffic(chunk, staged):
    """ncu DRAM bytes of one replay call on `chunk` events (captured at 2^26 events, scaled linearly)."""
    names = ("k_rpA<0>", "k_rpB") if staged else ("k_replay4",)
    tr = [load_traffic(k) for k in names]
    if any(t is None for t in tr):
        return None
    return sum(t["traffic_bytes_per_launch"] for t in tr) / 67108864 * chunk


def run_replay(args, torch, nb, dr, rank, world, local, peaks, peaks_src):
    dev = torch.device("cuda", local)
    wl = ReplayBench(torch, nb, dr, world, rank, n_total=args.replay_events, staged=args.replay_impl == "staged")
    evs = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
    # warm-up on one chunk
    for _ in range(args.warmup):
        nb.nvbt_gen_events(wl.ctx, 0x4E5642544E564254, 0, min(wl.chunk, wl.n), wl.hdr, wl.addr)
        wl.replay(min(wl.chunk, wl.n))
    nb.nvbt_reset(wl.ctx)
    torch.cuda.synchronize()
    barrier(world)
    l0 = nb.nvbt_launch_count(wl.ctx)
    with ClockSampler(local) as clk:
        ts = [wl.run(evs) for _ in range(args.steps)]
        if world > 1:
            dr.merge(wl.ctx)
        torch.cuda.synchronize()
        barrier(world)
    launches = nb.nvbt_launch_count(wl.ctx) - l0
    per, tot, hs, hl = nb.nvbt_mem_divergence(wl.ctx)
    cnt = nb.nvbt_count(wl.ctx)
    t_total = max_over_ranks(sum(ts), world, dev)
    n_all = wl.n * world if world > 1 else wl.n
    value = args.steps * sum_over_ranks(wl.n, world, dev) / t_total
    # algorithmic bytes: 16 B per header + 256 B per executed memory event (slots that must be read)
    mem_exec = int(tot[0]) // max(1, world if world > 1 else 1)
    bytes_rank = 16 * wl.n + 256 * (mem_exec // args.steps)
    ach = bytes_rank * args.steps / (sum(ts))
    line = {
        "metric": "replayed warp-instr events/sec", "value": value, "unit": "events/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_total / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": wl.desc.replace("10^10", f"{args.replay_events:.3g}" if args.replay_events != 10**10 else "10^10"),
                   "events": args.replay_events, "chunk": wl.chunk,
                   "l2": "inputs (36.5 GB per chunk) larger than L2"},
        "roofline": {"bound": "hbm", "achieved": ach / 1e9, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                     "frac": ach / 1e9 / peaks["hbm_gbs"], "peak_source": peaks_src,
                     "algorithmic_bytes_per_launch": bytes_rank * wl.chunk / wl.n,
                     "traffic": _replay_traffic(wl.chunk, staged=wl.scratch is not None),
                     "traffic_unit": "DRAM bytes per 2^27-event replay call (ncu at 2^26, scaled; profiles/r1_traffic.json)",
                     "kernel": "nvbt_replay_staged = k_rpA (headers, list) + k_rpB (slots)" if wl.scratch is not None
                     else "k_replay4"},
        "ncu_per_event": {"k_rpA": load_counters("k_rpA"), "k_rpB": load_counters("k_rpB"),
                          "source": "profiles/r1_ncu_counters.json (ncu --set full, tools/prof_step.py c5)"},
        "gpu_launches": int(launches), "clocks": clk.summary(),
        "check": {"W_issued": int(cnt[2]), "expected": args.steps * n_all},
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, sample = wl.oracle_sample(min(args.cpu_budget, 10.0))
        line["cpu_baseline"] = {"value": rate, "unit": "events/s", "cores": 1, "kind": "oracle", "sample": sample}
    if rank == 0:
        print(json.dumps(line), flush=True)



# --------------------------------------------------------------------------- C1 / C3 / C4 (profiling lines)
def _timed_events(torch, fn, n):
    ts = []
    for _ in range(n):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    return ts


def run_c1(args, torch, nb, dr, local):
    """C1: vectorAdd N = 65536, tools COUNT (instruction count + opcode histogram); a step is one launch.
    A launch moves 786 KB, so launch overhead dominates: the launches are batched into one CUDA graph of
    `reps` launches (captured on the context's stream) and each replay is timed."""
    from synth import uniform_f32
    N = 65536
    s = torch.cuda.Stream()
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT | nb.OPHIST | nb.BB, stream=s)
    a = torch.from_numpy(uniform_f32(N, 1)).cuda()
    b = torch.from_numpy(uniform_f32(N, 2)).cuda()
    c = torch.empty_like(a)
    reps = 200   # launches per graph
    torch.cuda.synchronize()

    def graph_of(tools):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(reps):
                nb.nvbt_vectoradd(ctx, tools, a, b, c, N)
        return g

    # per-pc counts two ways, identical results (I-5): a hook at every instruction (COUNT) or at block
    # leaders and guarded pcs only (BBCOUNT, the paper's basic-block instrumentation)
    g_plain, g_cnt, g_bb = graph_of(nb.TOOL_NONE), graph_of(nb.TOOL_COUNT), graph_of(nb.TOOL_BBCOUNT)
    nb.nvbt_reset(ctx)

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

    for g in (g_cnt, g_bb, g_plain):
        timed(g, args.warmup)
    tp = timed(g_plain, args.steps)
    res = {}
    for name, g in (("COUNT", g_cnt), ("BBCOUNT", g_bb)):
        nb.nvbt_reset(ctx)
        with ClockSampler(local) as clk:
            ti = timed(g, args.steps)
        cnt = nb.nvbt_count(ctx)
        ht, hw = nb.nvbt_opcode_hist(ctx)
        res[name] = (ti, cnt, ht, hw, clk.summary())
    ok = all((res["COUNT"][1] == res["BBCOUNT"][1]).all() and (res["COUNT"][k] == res["BBCOUNT"][k]).all()
             for k in (2, 3))
    ti, cnt, _, _, clocks = res["BBCOUNT"]
    ev = int(cnt[2]) // (args.steps * reps)
    t_i, t_p = sum(ti) / (args.steps * reps), sum(tp) / (args.steps * reps)
    t_c = sum(res["COUNT"][0]) / (args.steps * reps)
    return {"metric": METRIC, "value": ev / t_i, "unit": "events/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * t_i, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": "C1 vectorAdd N=65536, instruction counts + opcode histogram (tools BBCOUNT)",
                       "launches_per_graph": reps, "warp_events_per_launch": ev,
                       "counts_check": ("ok" if ev == 26624 else f"{ev} != 26624") +
                                       ("; COUNT == BBCOUNT counts and opcode histograms" if ok else "; COUNT != BBCOUNT")},
            "slowdown": t_i / t_p, "plain_us_per_launch": 1e6 * t_p, "instr_us_per_launch": 1e6 * t_i,
            "per_instruction_hooks": {"tools": "COUNT", "instr_us_per_launch": 1e6 * t_c, "slowdown": t_c / t_p,
                                      "value": ev / t_c},
            "bound": "launch latency (26,624 warp events per launch; CUDA-graph replays)", "clocks": clocks}


def run_c3(args, torch, nb, dr, local):
    """C3: BFS on an R-MAT scale-20 graph with BB-entry counting; a step is one whole BFS."""
    from synth import rmat_csr, bfs_source
    rowptr, col = rmat_csr(args.bfs_scale, 16, seed=3)
    n = len(rowptr) - 1
    src = bfs_source(rowptr)
    rp, cl = torch.from_numpy(rowptr).cuda(), torch.from_numpy(col).cuda()
    ctx = nb.nvbt_init(nb.W_BFS, nb.COUNT | nb.BB)
    bufs = dr.bfs_buffers(n, "cuda")
    f_plain = lambda: dr.run_bfs(ctx, nb.TOOL_NONE, rp, cl, src, bufs)
    f_instr = lambda: dr.run_bfs(ctx, nb.TOOL_BBCOUNT, rp, cl, src, bufs)
    for _ in range(args.warmup):
        f_plain(); f_instr()
    tp = _timed_events(torch, f_plain, args.steps)
    nb.nvbt_reset(ctx)
    with ClockSampler(local) as clk:
        ti = _timed_events(torch, f_instr, args.steps)
    cnt = nb.nvbt_count(ctx)
    ev = int(cnt[2]) // args.steps
    _, levels = f_plain()
    return {"metric": METRIC, "value": ev * args.steps / sum(ti), "unit": "events/s", "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(ti) / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"C3 BFS R-MAT scale {args.bfs_scale} ef16, tools BBCOUNT",
                       "vertices": n, "directed_edges": int(len(col)), "levels": levels,
                       "warp_events_per_bfs": ev},
            "slowdown": sum(ti) / sum(tp), "plain_ms_per_bfs": 1e3 * sum(tp) / args.steps,
            "bound": "latency of the hub warp's serial edge loop", "clocks": clk.summary()}


def run_c4(args, torch, nb, dr, local):
    """C4: 8192^2 5-point stencil x 100 iterations, every global LD/ST traced through the channel and
    drained to pinned host memory (digest callback on all host cores); a step is the whole run."""
    from synth import uniform_f32
    n, iters = args.stencil_n, args.stencil_iters
    ctx = nb.nvbt_init(nb.W_STENCIL, nb.COUNT | nb.TRACE)
    x0 = torch.from_numpy(uniform_f32((n, n), 4)).cuda()
    buf0, buf1 = x0.clone(), torch.empty_like(x0)
    slot = 176 if args.compact else 288
    ring = torch.empty(nb.nvbt_channel_bytes(args.ring_records, compact=args.compact), dtype=torch.uint8, pin_memory=True)
    ch = nb.nvbt_channel_open(ctx, ring, compact=args.compact)
    # plain baseline
    for _ in range(args.warmup):
        dr.run_stencil(ctx, nb.TOOL_NONE, buf0, buf1, n, iters)
    tp = _timed_events(torch, lambda: dr.run_stencil(ctx, nb.TOOL_NONE, buf0, buf1, n, iters), args.steps)
    # traced runs: wall time from first launch to the last record drained
    res = []
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dr.run_stencil(ctx, nb.TOOL_TRACE, buf0, buf1, n, iters)
            e1.record()
            if args.drain == "discard":
                nrec = nb.nvbt_channel_drain_discard(ch, timeout_us=600_000_000)
            else:
                nrec = nb.nvbt_channel_drain_digest(ch, timeout_us=600_000_000).n_rec
            torch.cuda.synchronize()
            res.append((time.perf_counter() - t0, nrec, e0.elapsed_time(e1) / 1e3))
    dropped = nb.nvbt_channel_dropped(ch)
    recs = res[-1][1]
    t_tr = sum(r[0] for r in res) / len(res)
    G = n // 32
    expect = iters * (2 * (n * n // 32) + 4 * (n - 2) * G)
    return {"metric": "traced warp-level memory events/sec (records drained to host)", "value": recs / t_tr,
            "unit": "records/s", "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_tr,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"C4 stencil {n}^2 x {iters}, tools TRACE", "ring_slots": args.ring_records,
                       "transport": "compact 176 B slots at a 192 B stride (EM 5.1)" if args.compact else "288 B records",
                       "host_callback": args.drain},
            "records_per_run": recs, "records_expected": expect, "dropped": dropped,
            "gpu_s_per_run": sum(r[2] for r in res) / len(res),
            "host_threads": os.environ.get("NVBT_DRAIN_THREADS", str(os.cpu_count())),
            "GB_per_s_to_host": recs * slot / t_tr / 1e9, "record_GB_per_s": recs * 288 / t_tr / 1e9, "slowdown": t_tr / (sum(tp) / len(tp)),
            "plain_ms": 1e3 * sum(tp) / len(tp), "bound": "PCIe D2H (measured 52.7 GB/s SM stores to pinned memory)",
            "clocks": clk.summary()}


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
                         "traffic_unit": "DRAM bytes per launch (ncu, profiles/r1_traffic.json)",
                         "algorithmic_bytes_per_launch": bytes_launch, "kernel": "k_wfft<EMU|COUNT, proxy>"},
            "sw_plain_hbm_frac": bytes_launch / med["sw_plain"] / 1e9 / hbm_peak,
            "clocks": clk.summary(), "peaks_source": peaks_src,
            "paper_context": "21 vs 150 instructions per warp with and without WFFT32 (P:L295), parity-unpinned"}


def run_reference(args):
    """Reference arm = the CPU oracle (this tier has no runnable reference)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import events as ev, programs
    from oracle.models import sgemm as m_sg
    M = N = K = 1024
    nw = (M // 32) * (N // 8) * 8
    events_per_launch = nw * (12 + 6 * K)
    base = 1 << 32
    rng = np.random.default_rng(1)
    warps = np.sort(rng.choice(nw, size=16, replace=False))
    per_step_events = len(warps) * (12 + 6 * K)
    for _ in range(args.warmup):
        acc = ev.Accumulator(programs.sgemm())
        m_sg.run(acc, M, N, K, base, base + (8 << 20), base + (16 << 20), warps=warps[:2])
    ts = []
    for _ in range(args.steps):
        acc = ev.Accumulator(programs.sgemm())
        t0 = time.perf_counter()
        m_sg.run(acc, M, N, K, base, base + (8 << 20), base + (16 << 20), warps=warps)
        ts.append(time.perf_counter() - t0)
    value = per_step_events * args.steps / sum(ts)
    sample = (f"{per_step_events} warp events per step: 16 sampled warps (full K) of C2 SGEMM 1024^3 "
              f"({events_per_launch} events per launch)")
    line = {
        "metric": METRIC, "value": value, "unit": "events/s", "n_gpus": int(os.environ.get("WORLD_SIZE", "1")),
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(ts) / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": SgemmBench.desc, "M": M, "N": N, "K": K}, "impl": "reference",
        "cpu_baseline": {"value": value, "unit": "events/s", "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "events/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--drain", choices=["digest", "discard"], default="digest",
                    help="C4: host callback (digest of every record, or discard: the transport alone)")
    ap.add_argument("--replay-impl", choices=["staged", "single"], default="staged",
                    help="C5: two-pass staged replay (default) or the single-pass kernel")
    ap.add_argument("--workload", choices=["c1", "c2", "c3", "c4", "c5", "f1", "f2", "f4"], default="c2")
    ap.add_argument("--fft-n", type=int, default=1 << 24, help="F4: transforms per launch")
    ap.add_argument("--fft-ctas", type=int, default=0, help="F4: grid (0 = one resident wave per kernel)")
    ap.add_argument("--f2-iters", type=int, default=10, help="F2: stencil iterations kept in the HBM ring")
    ap.add_argument("--bfs-scale", type=int, default=20)
    ap.add_argument("--stencil-n", type=int, default=8192)
    ap.add_argument("--stencil-iters", type=int, default=100)
    ap.add_argument("--ring-records", type=int, default=1 << 22)
    ap.add_argument("--compact", action="store_true", help="C4: compact 176 B transport slots (F3)")
    ap.add_argument("--replay-events", type=int, default=10**10)
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
