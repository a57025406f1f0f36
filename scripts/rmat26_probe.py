#!/usr/bin/env python
"""Feasibility probe for configs[4] (RMAT scale 26, ~1B edges): device
generation, fsgc_load_graph, then one count per pattern group with timings.
    python scripts/rmat26_probe.py [scale] [patterns]"""
import os
import sys
import time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS
from inputs.graphs import rmat_edges_torch

sc = int(sys.argv[1]) if len(sys.argv) > 1 else 26
groups = (sys.argv[2] if len(sys.argv) > 2 else "tricore+1f;tricore+1f,tricore+2f,tricore+3f,tricore+4f,tricore+5f,tricore+6f").split(";")
t0 = time.time()
e = rmat_edges_torch(sc, 16, seed=6, device="cuda")
torch.cuda.synchronize()
print(f"gen scale {sc}: {e.shape[0]} raw edges {time.time()-t0:.1f}s", flush=True)
t0 = time.time()
g = F.fsgc_load_graph(e, 1 << sc)
torch.cuda.synchronize()
del e
torch.cuda.empty_cache()
print(f"load {time.time()-t0:.1f}s n={g.n} m={g.m} dmax={g.max_degree} mem={torch.cuda.max_memory_allocated()/2**30:.1f}GiB", flush=True)
for grp in groups:
    names = grp.split(",")
    ps = [F.compile_named(PATTERNS[x]) for x in names]
    for rep in range(2):
        t0 = time.time()
        res = F.fsgc_count(g, ps)
        torch.cuda.synchronize()
        print(f"rep{rep} {time.time()-t0:.2f}s", {x: (r.count, round(r.kernel_ms, 1), round(r.aux_ms, 1)) for x, r in zip(names, res)}, flush=True)
