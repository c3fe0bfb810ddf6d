"""Helpers for the GPU parity tests: run the CUDA path through the C ABI, read every result, and compare
it with the oracle element by element (bit-exact: all of this work is integer, EM §2)."""
import numpy as np

from oracle import events as ev


def read_all(nb, ctx, per_warp=False):
    r = {}
    if per_warp:
        c, pwt, pww = nb.nvbt_count(ctx, per_warp=True)
        r["PW_T"], r["PW_W"] = pwt.astype(np.int64), pww.astype(np.int64)
    else:
        c = nb.nvbt_count(ctx)
    r["counts"] = c.astype(np.int64)
    t, w = nb.nvbt_opcode_hist(ctx)
    r["H_t"], r["H_w"] = t.astype(np.int64), w.astype(np.int64)
    bb = nb.nvbt_bb_count(ctx).astype(np.int64)
    r["Ent_w"], r["Ent_t"], r["Ins_w"], r["Ins_t"] = bb[:, 0], bb[:, 1], bb[:, 2], bb[:, 3]
    if ctx.flags & nb.MEMDIV:
        per, tot, hs, hl = nb.nvbt_mem_divergence(ctx)
        per = per.astype(np.int64)
        r["mem_n"], r["mem_S"], r["mem_L"] = per[:, 0], per[:, 1], per[:, 2]
        r["hS"], r["hL"] = hs.astype(np.int64), hl.astype(np.int64)
        assert (tot.astype(np.int64) == per.sum(axis=0)).all()
    return r


def assert_same(gpu, ref, keys=None, what=""):
    keys = keys or [k for k in gpu if k in ref]
    for k in keys:
        g, o = np.asarray(gpu[k]), np.asarray(ref[k])
        if g.shape != o.shape or not (g == o).all():
            idx = np.nonzero(g != o)[0] if g.shape == o.shape else []
            raise AssertionError(f"{what}: {k} differs (first index {idx[:5]}): gpu {g[idx[:5]] if len(idx) else g} "
                                 f"oracle {o[idx[:5]] if len(idx) else o}")


def gpu_invariants(r):
    bad = ev.invariants({**r, **({} if "mem_n" in r else {
        "mem_n": np.zeros(1, np.int64), "mem_S": np.zeros(1, np.int64), "mem_L": np.zeros(1, np.int64),
        "hS": np.zeros(33, np.int64), "hL": np.zeros(33, np.int64)})})
    assert bad == [], bad
