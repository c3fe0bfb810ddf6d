"""C-ABI library checks that need no GPU: it loads, exports every symbol include/*.h declares, and its
host-only entry points behave (program tables, sizes, argument validation, host digest)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_micro_villasnk19_b200", "libnvbt.so")
pytestmark = pytest.mark.skipif(not os.path.exists(LIB), reason="libnvbt.so not built")


def declared_symbols():
    names = set()
    for h in ("nvbt.h", "nvbt_workloads.h"):
        txt = open(os.path.join(ROOT, "include", h)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        names |= set(re.findall(r"\b(nvbt_[a-z0-9_]+)\s*\(", txt))
    return names - {"nvbt_drain_fn"}


def test_every_declared_symbol_is_exported():
    lib = C.CDLL(LIB)
    names = declared_symbols()
    assert len(names) >= 25
    missing = [n for n in sorted(names) if not hasattr(lib, n)]
    assert missing == []


def test_binding_covers_declared_symbols():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    assert declared_symbols() <= set(nb.EXPORTED)
    assert nb.nvbt_abi_version() == 1


@pytest.mark.parametrize("w,name", [(1, "vectoradd"), (2, "sgemm"), (3, "bfs"), (4, "stencil"), (5, "replay")])
def test_program_tables_match_oracle_transcription(w, name):
    """Both sides transcribe docs/EVENT_MODEL.md §3 independently; the tables must agree."""
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import programs
    arr, n_ops, n_bbs = nb.nvbt_program(w)
    got = nb.program_numpy(arr)
    exp = getattr(programs, name)()
    assert n_ops == exp["n_opcodes"] and n_bbs == exp["n_bbs"] and len(arr) == exp["n_pcs"]
    for k in got:
        assert (got[k] == exp[k]).all(), k


def test_workspace_and_validation_errors():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    assert nb.nvbt_workspace_size(18, 16, 4, nb.COUNT) > 0
    big = nb.nvbt_workspace_size(18, 16, 4, nb.COUNT | nb.PER_WARP, n_warps=1 << 20)
    assert big >= 16 * (1 << 20)
    with pytest.raises(nb.NvbtError) as e:
        nb.nvbt_workspace_size(0, 16, 4, nb.COUNT)
    assert e.value.code == nb.EINVAL
    with pytest.raises(nb.NvbtError):
        nb.nvbt_workspace_size(18, 16, 4, nb.PER_WARP)   # PER_WARP needs n_warps
    with pytest.raises(nb.NvbtError):
        nb.nvbt_workspace_size(18, 16, 4, 1 << 9)        # unknown flag
    assert nb.nvbt_workload_warps(nb.W_SGEMM, 1024, 1024) == 32768
    assert nb.nvbt_workload_warps(nb.W_VECTORADD, 65500) == 2048
    assert nb.nvbt_workload_warps(nb.W_STENCIL, 8192) == 2097152


def test_host_digest_matches_oracle():
    from paper_conf_micro_villasnk19_b200 import nvbt as nb
    from oracle import events as ev, programs, trace
    from oracle.models import stencil
    acc = ev.Accumulator(programs.stencil(), trace=True, keep_records=True)
    stencil.run(acc, 64, 1 << 32, (1 << 32) + (1 << 24))
    recs = acc.record_array()
    assert nb.nvbt_digest_records(recs) == (acc.digest.n, acc.digest.d1, acc.digest.d2)
