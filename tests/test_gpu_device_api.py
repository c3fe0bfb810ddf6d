"""The public device API (include/nvbt_dev.cuh + nvbt_device_state): a kernel compiled OUTSIDE
libnvbt.so (tests/ext/ext_gather.cu, nvcc'd here against include/ only) instruments itself with
nvbt_on_instr / nvbt_on_bb / nvbt_on_mem / nvbt_cta_flush, and the context's read calls report, bit-exactly,
what the oracle computes for the same events (docs/EVENT_MODEL.md §2). The compiled-in analogue of
nvbit_insert_call / nvbit_add_call_arg on someone else's kernel (P:L123 (§4); Listing 8)."""
import ctypes as C
import os
import subprocess

import numpy as np
import pytest

from oracle import events as ev, programs
from oracle.models import mask_of, FULL

from .gpu_util import read_all, assert_same, gpu_invariants

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tests", "ext", "ext_gather.cu")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
S2R, ISETP, EXIT, LDG, STG, FFMA = (programs.S2R, programs.ISETP, programs.EXIT, programs.LDG, programs.STG,
                                     programs.FFMA)
A_, C_, GLD, GST = programs.ALU, programs.CTRL, programs.GLD, programs.GST
# (opcode, kind, width, bb, is_leader, guarded) — the table ext_gather.cu's header states
PROGRAM = [(S2R, A_, 0, 0, 1, 0), (ISETP, A_, 0, 0, 0, 0), (EXIT, C_, 0, 0, 0, 1),
           (LDG, GLD, 4, 1, 1, 0), (LDG, GLD, 4, 1, 0, 1), (FFMA, A_, 0, 1, 0, 0), (STG, GST, 4, 1, 0, 0),
           (EXIT, C_, 0, 1, 0, 0)]
COUNT_KEYS = ["counts", "H_t", "H_w", "Ent_w", "Ent_t", "Ins_w", "Ins_t"]
MEM_KEYS = ["mem_n", "mem_S", "mem_L", "hS", "hL"]


def build_ext(out_dir, check_converged=True):
    """nvcc against include/ only; with check_converged every hook traps unless the whole warp reached it
    (NVBT_CHECK_CONVERGED, the converged-hook discipline R-15)."""
    so = os.path.join(out_dir, "libext_gather.so")
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           *(["-DNVBT_CHECK_CONVERGED"] if check_converged else []),
           "-I", os.path.join(ROOT, "include"), SRC, "-o", so]
    r = subprocess.run(cmd, capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr
    return so


def test_public_header_compiles_standalone(tmp_path):
    """CPU-side check: the public header alone is enough to build an instrumented kernel for sm_100a."""
    if not os.path.exists(NVCC):
        pytest.skip("no nvcc")
    build_ext(str(tmp_path))


def oracle_prog():
    cols = list(zip(*PROGRAM))
    p = {k: np.array(v, dtype=np.int64) for k, v in zip(("opcode", "kind", "width", "bb", "is_leader", "guarded"), cols)}
    p.update(n_pcs=len(PROGRAM), n_opcodes=programs.N_OPCODES_WL, n_bbs=2)
    return p


def oracle_run(acc, idx, n, idx_p, x_p, y_p, block):
    """EM §1-2 events of ext_gather (lane = i % 32, warp w covers i = 32 w .. 32 w + 31)."""
    nw = -(-n // block) * (block // 32)
    warps = np.arange(nw)
    i = warps[:, None] * 32 + np.arange(32)[None, :]
    full = np.full(nw, FULL)
    acc.add(0, warps, 0, full, full)
    acc.add(0, warps, 1, full, full)
    acc.add(0, warps, 2, full, mask_of(i >= n))
    live = i < n
    A = mask_of(live)
    k = np.where(live, idx[np.minimum(i, n - 1)], 0)
    p1 = live & (k % 3 != 0)
    u = lambda base, off: np.uint64(base) + (off * 4).astype(np.uint64)
    acc.add(0, warps, 3, A, A, u(idx_p, i))
    acc.add(0, warps, 4, A, mask_of(p1), u(x_p, k))
    acc.add(0, warps, 5, A, A)
    acc.add(0, warps, 6, A, A, u(y_p, i))
    acc.add(0, warps, 7, A, A)


@pytest.fixture(scope="module")
def ext(tmp_path_factory):
    lib = C.CDLL(build_ext(str(tmp_path_factory.mktemp("ext"))))
    lib.ext_gather_launch.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_int, C.c_void_p]
    lib.ext_gather_launch.restype = C.c_int
    return lib


@pytest.mark.gpu
@pytest.mark.parametrize("n,block,spread", [(5000, 256, 64), (1 << 16, 128, 1 << 20), (777, 64, 1 << 26), (32, 32, 8)])
@pytest.mark.parametrize("tools", ["COUNT|MEMDIV", "BBCOUNT|MEMDIV", "BBCOUNT"])
def test_external_kernel_matches_oracle(nvbt, ext, n, block, spread, tools):
    import torch
    nb = nvbt.nvbt
    t = 0
    for x in tools.split("|"):
        t |= getattr(nb, "TOOL_" + x)
    arr = (nb.InstrDesc * len(PROGRAM))(*[nb.InstrDesc(o, k, w, b, l, g, 0) for o, k, w, b, l, g in PROGRAM])
    nw = -(-n // block) * (block // 32)
    ctx = nb.nvbt_init(arr, nb.COUNT | nb.OPHIST | nb.BB | nb.MEMDIV | nb.PER_WARP, n_warps=nw,
                       n_opcodes=programs.N_OPCODES_WL, n_bbs=2)
    rng = np.random.default_rng(n)
    idx_h = rng.integers(0, spread, n).astype(np.int32)         # gather spread: one word .. 256 MB
    idx = torch.from_numpy(idx_h).cuda()
    x = torch.from_numpy(rng.random(spread).astype(np.float32)).cuda()
    y = torch.zeros(n, device="cuda")
    st = nb.nvbt_device_state(ctx, t)
    assert st.version == 1 and st.n_pcs == len(PROGRAM) and st.n_warps == nw
    rc = ext.ext_gather_launch(C.byref(st), idx.data_ptr(), x.data_ptr(), y.data_ptr(), n, block,
                               torch.cuda.current_stream().cuda_stream)
    assert rc == 0
    g = read_all(nb, ctx, per_warp=True)
    acc = ev.Accumulator(oracle_prog(), n_warps=nw)
    oracle_run(acc, idx_h, n, idx.data_ptr(), x.data_ptr(), y.data_ptr(), block)
    keys = COUNT_KEYS + ["PW_T", "PW_W"] + (MEM_KEYS if "MEMDIV" in tools else [])
    assert_same(g, acc.result(), keys, f"external gather n={n} {tools}")
    gpu_invariants(g)
    k = idx_h
    ref = np.where(k % 3 != 0, 2 * x.cpu().numpy()[k] + 1, 1).astype(np.float32)
    assert np.array_equal(y.cpu().numpy(), ref)


@pytest.mark.gpu
def test_device_state_errors(nvbt):
    nb = nvbt.nvbt
    ctx = nb.nvbt_init(nb.W_VECTORADD, nb.COUNT)
    with pytest.raises(nb.NvbtError):
        nb.nvbt_device_state(ctx, nb.TOOL_TRACE)                 # not offered to external kernels
    with pytest.raises(nb.NvbtError):
        nb.nvbt_device_state(ctx, nb.TOOL_MEMDIV)                # MEMDIV not enabled at init
    with pytest.raises(nb.NvbtError):
        nb.nvbt_device_state(ctx, nb.TOOL_COUNT | nb.TOOL_BBCOUNT)
