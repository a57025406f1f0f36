"""Fringe-SGC ORACLE -- test infrastructure, NOT part of the product.

Plain, slow, obviously-correct CPU implementation of what the CUDA path
computes, written from PAPER.md (Bradley, Alabandi, Burtscher, "Fringe-SGC:
Counting Subgraphs with Fringe Vertices", SC'25).  Python integers (exact,
unbounded) are used for every count.  Only ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with ``paper_conf_sc_bradleyab25_b200`` and never
imports it; its inputs come from ``inputs/`` (generators only).

Modules
  graph    simple undirected graph from an edge list; degree-ordered CSR
           (the definition the product's ``fsgc_load_graph`` must reproduce)
  pattern  Sec. 3.4 core/fringe decomposition heuristic, anchor sets
           (Def. 3.1-3.3), fringe grouping, automorphism count (Sec. 3.1)
  count    mode 1: brute-force monomorphism enumeration of the whole pattern
           divided by |Aut(P)|; mode 2: core-plus-fringe counting -- enumerate
           core matches, Venn diagram of external neighbours (Sec. 3.3-3.4),
           fringe counting function fc (Listing 5), scaled by the fringe
           multiplicities and divided by |Aut(P)|.

  cfast    mode 2 with the per-core-map work (Venn by explicit marking,
           Listing 5) in plain C (oracle/c/core_fringe.c, gcc -fopenmp):
           the same definition, fast enough for RMAT graphs with hubs;
           pinned to the Python oracle and to closed forms.

Pins (tests/test_oracle.py, ``-m "not gpu"``): Fig. 2 facts, closed forms
(k-stars, wedges, trace(A^3)/6, trace(A^4) 4-cycles, tailed triangles), Sec. 3.1
explicit edge-core formulas, definition-level brute force of fc on explicit
sets, exhaustive mode-1 vs mode-2 on all connected patterns <= 5 vertices and
all graphs <= 5 vertices, known automorphism counts.  Every function here is
pinned; none is "parity unpinned".
"""
from .graph import simple_adjacency, degree_ordered_csr, csr_to_adjacency  # noqa: F401
from .pattern import (  # noqa: F401
    pattern_adjacency, automorphism_count, decompose, Decomposition,
)
from .count import (  # noqa: F401
    count_monomorphisms, brute_force_count, fc, venn_sizes, fringe_count,
    core_matches, root_raw_sum, closed_forms, k_tailed_triangles,
)
