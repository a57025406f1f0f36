#!/usr/bin/env python
"""Count patterns on a workload under the current FSGC_* environment and print
raw values (compare runs with different tuning knobs).
    python scripts/debug_variants.py WORKLOAD|rmatSC p1,p2,.. [reps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch

import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS, workload_edges
from inputs.graphs import rmat_edges_torch

wl, names = sys.argv[1], sys.argv[2].split(",")
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
if wl.startswith("rmat") and wl.endswith("x"):      # rmatSCx: edge factor 16, seed 5
    sc = int(wl[4:-1])
    n, e = 1 << sc, rmat_edges_torch(sc, 16, seed=5, device="cuda")
else:
    n, e = workload_edges(wl)
g = F.fsgc_load_graph(e, n)
env = {k: v for k, v in os.environ.items() if k.startswith("FSGC_")}
for nm in names:
    p = F.compile_named(PATTERNS[nm])
    for r in range(reps):
        x = F.fsgc_count(g, [p], no_symmetry_breaking=False)[0]
        print(f"{env} {nm} rep{r}: raw={x.raw} ovf={x.overflow} div={x.divisor} kind={x.pass_kind}", flush=True)
