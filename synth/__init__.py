"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the CPU oracle.

This package holds NO arithmetic of the method (no masks, counts, histograms, divergence or trace
logic): only the raw inputs the synthetic workloads consume — fp32 operand arrays (their values do not
affect any event) and the R-MAT graph for the BFS workload (C3). Recipes are stated in DESIGN.md §6.
The C5 replay events are NOT generated here: each side implements the counter-based generator of
docs/EVENT_MODEL.md §3.5 independently.
"""
from .inputs import uniform_f32, rmat_csr, bfs_source  # noqa: F401
