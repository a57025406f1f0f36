"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This package holds ONLY input generation (graphs as raw edge lists, patterns as
small edge lists).  It contains none of Fringe-SGC's arithmetic: no CSR build,
no core/fringe decomposition, no counting.  Both ``oracle/`` and
``paper_conf_sc_bradleyab25_b200`` consume its outputs; neither is imported here.
"""
from .rng import splitmix64_np, counter_u64_np, counter_u64_torch  # noqa: F401
from .graphs import (  # noqa: F401
    fig2_edges, powerlaw_edges, rmat_edges_np, rmat_edges_torch, WORKLOADS,
    workload_edges,
)
from .patterns import PATTERNS, Pattern, get_pattern  # noqa: F401
