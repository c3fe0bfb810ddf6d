"""Builds libnvbt.so in-tree for sm_100a (nvcc). `python -m paper_conf_micro_villasnk19_b200.build`."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
SOURCES = ["nvbt_core.cu", "channel.cu", "workloads.cu", "replay.cu", "wfft.cu"]
OUT = os.path.join(HERE, "libnvbt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
         "-Xcompiler", "-fPIC,-O3,-march=x86-64-v3", "-shared"]


DEBUG_OUT = os.path.join(HERE, "libnvbt_debug.so")
# the debug build: every hook checks the converged-hook discipline (__activemask() == all lanes, else trap)
DEBUG_DEFS = ["-DNVBT_CHECK_CONVERGED"]


def _stale(out):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [
        os.path.join(ROOT, "include", f) for f in os.listdir(os.path.join(ROOT, "include"))]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(out, defs, tag):
    objs = []
    procs = []
    for src in SOURCES:
        obj = os.path.join(CSRC, src.replace(".cu", f"{tag}.o"))
        cmd = [NVCC, *FLAGS[:-1], *defs, "-c", "-I", os.path.join(ROOT, "include"), "-I", CSRC,
               os.path.join(CSRC, src), "-o", obj]
        procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        objs.append(obj)
    return procs, objs


def _link(out, procs, objs, verbose):
    for src, p in procs:
        o, _ = p.communicate()
        if p.returncode != 0:
            raise RuntimeError(f"nvcc failed on {src}:\n{o.decode()}")
        if verbose and o.strip():
            print(o.decode(), file=sys.stderr)
    tmp = out + ".tmp"
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", *objs, "-o", tmp]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}{r.stderr}")
    os.replace(tmp, out)
    for o in objs:
        os.remove(o)
    if verbose:
        print(f"built {out}", file=sys.stderr)


def build(force: bool = False, verbose: bool = True, debug: bool = True) -> str:
    """Builds libnvbt.so (and, with debug, libnvbt_debug.so) in-tree; both compile in parallel."""
    jobs = []
    if force or _stale(OUT):
        jobs.append((OUT, *_compile(OUT, [], "")))
    if debug and (force or _stale(DEBUG_OUT)):
        jobs.append((DEBUG_OUT, *_compile(DEBUG_OUT, DEBUG_DEFS, "_dbg")))
    for out, procs, objs in jobs:
        _link(out, procs, objs, verbose)
    return OUT


if __name__ == "__main__":
    build(force="--force" in sys.argv)
