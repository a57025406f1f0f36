#!/usr/bin/env python
"""Match-count census of the RMAT workloads (readings R14/R15):
m, max degree, wedges sum C(d, 2), 2-paths through edges sum C(c(e), 2) is
the diamond count (measured by the counting path instead).
    python scripts/census.py 16 18 20 22 26"""
import os
import sys
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from inputs.graphs import rmat_edges_torch, workload_edges

for sc in [int(x) for x in sys.argv[1:]]:
    n = 1 << sc
    if sc in (22, 26):
        _, e = workload_edges(f"rmat{sc}", device="cuda")
    else:
        e = rmat_edges_torch(sc, 16, seed=5, device="cuda")
    e = e.to(torch.int64)
    a = torch.minimum(e[:, 0], e[:, 1]); b = torch.maximum(e[:, 0], e[:, 1])
    del e
    ok = a != b
    k = torch.unique(a[ok] * n + b[ok])
    del a, b, ok
    deg = torch.bincount(k // n, minlength=n) + torch.bincount(k % n, minlength=n)
    d = deg.to(torch.float64)
    wedges = int((deg * (deg - 1) // 2).sum())
    print(f"RMAT-{sc}: n {n} m {k.numel()} max_degree {int(deg.max())} wedges {wedges:.4e} "
          f"sum d^2 {float((d * d).sum()):.4e}", flush=True)
    del k, deg, d
    torch.cuda.empty_cache()
