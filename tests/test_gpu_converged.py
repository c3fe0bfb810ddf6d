"""Converged-hook discipline (R-15, SURVEY §4 plan item 2): every hook must be reached by all 32 lanes
of the warp (lanes outside the flow pass in_flow = false). libnvbt_debug.so is the same library built
with NVBT_CHECK_CONVERGED, where each hook traps unless __activemask() is the full warp. The GPU parity
suites run again in a subprocess against that build (NVBT_LIB): any divergent hook call would trap the
kernel and fail them, and every result must still match the oracle."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
DEBUG_LIB = os.path.join(ROOT, "paper_conf_micro_villasnk19_b200", "libnvbt_debug.so")


@pytest.mark.gpu
def test_parity_suites_under_converged_hook_checks():
    assert os.path.exists(DEBUG_LIB), "libnvbt_debug.so not built (__graft_entry__.build())"
    env = dict(os.environ, NVBT_LIB=DEBUG_LIB)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_gpu_parity.py"), os.path.join(ROOT, "tests", "test_gpu_wfft.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout


def test_debug_library_loads_and_exports_the_abi():
    """CPU check: the debug build exists beside the release build and exports the same ABI version."""
    import ctypes
    if not os.path.exists(DEBUG_LIB):
        pytest.skip("libnvbt_debug.so not built")
    lib = ctypes.CDLL(DEBUG_LIB)
    assert lib.nvbt_abi_version() == 1
