#!/usr/bin/env python
"""Per-edge support statistics of a workload (design input for the 4-clique
core kernels): sum c(e) = 3 T, sum c(e)^2 (pair work of a 4-clique listing
from the common out-neighbourhoods), max c(e).  python scripts/sup_stats.py WL"""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS, workload_edges
from inputs.graphs import rmat_edges_torch
for wl in sys.argv[1:]:
    if wl.startswith("rmat") and wl.endswith("x"):
        sc = int(wl[4:-1])
        n, e = 1 << sc, rmat_edges_torch(sc, 16, seed=5, device="cuda")
    else:
        n, e = workload_edges(wl, device="cuda") if wl.startswith("rmat") else workload_edges(wl)
    g = F.fsgc_load_graph(e, n)
    plan = F.Plan(g, [F.compile_named(PATTERNS["2-tailed-triangle"])])
    plan.enqueue()
    torch.cuda.synchronize()
    s = plan.support().to(torch.float64)
    print(wl, {"m": g.m, "triangles": float(s.sum()) / 3, "sum_c2": float((s * s).sum()),
               "sum_c3": float((s ** 3).sum()), "max_c": float(s.max())}, flush=True)
