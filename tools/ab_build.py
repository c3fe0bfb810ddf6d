"""Builds A/B variants of libnvbt.so with extra -D flags, for tools/replay_ab.py (never product builds).

usage: python tools/ab_build.py TAG [-DNAME=VALUE ...] [TAG2 -D... ...]
       each TAG is built as ab/libnvbt_TAG.so from the current sources with the flags that follow it."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_micro_villasnk19_b200 import build as b  # noqa: E402


def main(argv):
    jobs, cur = [], None
    for a in argv:
        if a.startswith("-D"):
            cur[1].append(a)
        else:
            cur = (a, [])
            jobs.append(cur)
    os.makedirs(os.path.join(ROOT, "ab"), exist_ok=True)
    started = []
    for tag, defs in jobs:
        out = os.path.join(ROOT, "ab", f"libnvbt_{tag}.so")
        procs, objs = b._compile(out, defs, f"_ab_{tag}")
        started.append((out, procs, objs))
    for out, procs, objs in started:
        b._link(out, procs, objs, True)


if __name__ == "__main__":
    main(sys.argv[1:])
