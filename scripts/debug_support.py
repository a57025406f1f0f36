#!/usr/bin/env python
"""Check the per-edge support array of a plan against c(e) <= min(deg)-1 and,
for a sample of edges (all violators first), against a direct intersection of
the downloaded CSR.   python scripts/debug_support.py SCALE [EF]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS
from inputs.graphs import rmat_edges_torch

sc = int(sys.argv[1])
ef = int(sys.argv[2]) if len(sys.argv) > 2 else 16
e = rmat_edges_torch(sc, ef, seed=5, device="cuda")
g = F.fsgc_load_graph(e, 1 << sc)
offs, adj, _ = g.download()
n = g.n
deg = np.diff(offs)
rows = np.repeat(np.arange(n), deg)
up = adj > rows
osrc, odst = rows[up], adj[up]
print(f"scale {sc} ef {ef}: n={n} m={g.m} dmax={g.max_degree}  oriented={len(osrc)}", flush=True)
p = F.compile_named(PATTERNS["4-tailed-triangle"])
plan = F.Plan(g, [p])
plan.enqueue()
torch.cuda.synchronize()
sup = plan.support().cpu().numpy().astype(np.int64)
res = plan.decode()[0]
print("4-tailed:", res.count, res.overflow, "sum sup", int(sup.sum()), flush=True)
lim = np.minimum(deg[osrc], deg[odst]) - 1
bad = np.nonzero(sup > lim)[0]
neg = np.nonzero(sup < 0)[0]
print(f"violations c > min(deg)-1: {len(bad)}, negative: {len(neg)}", flush=True)
rng = np.random.default_rng(0)
sample = list(bad[:20]) + list(rng.choice(len(osrc), 200, replace=False))
wrong = 0
for i in sample:
    u, v = osrc[i], odst[i]
    a = adj[offs[u]:offs[u + 1]]
    b = adj[offs[v]:offs[v + 1]]
    c = len(np.intersect1d(a, b, assume_unique=True))
    if c != sup[i]:
        wrong += 1
        if wrong <= 10:
            print(f"  edge {i} ({u},{v}) deg {deg[u]},{deg[v]} out {np.sum(a > u)},{np.sum(b > v)}: gpu {sup[i]} true {c}",
                  flush=True)
print(f"sampled {len(sample)} edges, wrong {wrong}", flush=True)
