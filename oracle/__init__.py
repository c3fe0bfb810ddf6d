"""nvbt CPU oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the nvbt hot path computes, written from
docs/EVENT_MODEL.md and the paper (/root/reference/PAPER.md; citations `P:Lnnn (§x)`). It shares no
code with the CUDA path (paper_conf_micro_villasnk19_b200/), and neither imports the other; the only
common dependency is `synth/` (seeded raw inputs, no method arithmetic).

Only `tests/`, `__graft_entry__.smoke()` and `bench.py` (its `cpu_baseline` leg and `--impl reference`)
may import anything under `oracle/`. The product path never routes through it.

Modules and their pins (tests/test_oracle_*.py):
  mix          splitmix64 finaliser        pinned: published splitmix64 output for seed 0, 2**64 wrap
  events       §2 per-event definitions    pinned: brute force over all (A, P) at warp widths 1..5 (I-1),
                                           Fraction identity of Listing 8's 1/cnt sums (C-5),
                                           numpy.unique / set definitions, invariants (I-2)
  programs     §3 program tables           pinned: BB rule checks (leaders after CTRL and at targets)
  models.*     §3.1-3.4 CPU workload models pinned: closed forms (I-3) for vectorAdd, SGEMM, stencil;
                                           BFS distances vs scipy.sparse.csgraph (I-4); invariants
  models.wfft  §3.6 F4 WFFT32 emulation    pinned: DFT vs numpy.fft.fft, single-exponential / constant /
                                           delta closed forms, Parseval, Hermitian symmetry, inverse
                                           round trip; per-warp count closed forms, BB identity (I-5)
  gen          §3.5 C5 generator           pinned: mix64 vector, distribution/alignment properties,
                                           partition invariance
  trace        §5 records + digests        pinned: record field layout by hand-built record,
                                           order independence, single-bit sensitivity
               footprint (F2)              pinned: Python-set brute force on random records, vectorAdd
                                           closed form 3*ceil(4N/32) sectors / 3*ceil(4N/128) lines
Parity unpinned: none of the above; the paper's Figs 5–9 values, the 74–96 % library share
and WFFT32's 21 vs 150 instructions/warp need the paper's kernels; §3.6 models our own pair.
"""
