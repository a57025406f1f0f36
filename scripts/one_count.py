#!/usr/bin/env python
"""One count of the given patterns on rmatSC (ef 16, seed 5) or a named
workload, repeated R times (for ncu launch lists).
    python scripts/one_count.py rmat20x|WORKLOAD p1,p2 [R]"""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS, workload_edges
from inputs.graphs import rmat_edges_torch
wl, names = sys.argv[1], sys.argv[2].split(",")
R = int(sys.argv[3]) if len(sys.argv) > 3 else 2
if wl.startswith("rmat") and wl.endswith("x"):
    sc = int(wl[4:-1])
    n, e = 1 << sc, rmat_edges_torch(sc, 16, seed=5, device="cuda")
else:
    n, e = workload_edges(wl, device="cuda") if wl.startswith("rmat") else workload_edges(wl)
g = F.fsgc_load_graph(e, n)
ps = [F.compile_named(PATTERNS[x]) for x in names]
for _ in range(R):
    res = F.fsgc_count(g, ps)
torch.cuda.synchronize()
print({x: (r.count, r.kernel_ms, r.aux_ms) for x, r in zip(names, res)})
