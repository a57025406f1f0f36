#!/usr/bin/env python
"""Degree-orientation statistics of the RMAT workloads (design input for the
support / triangle-core kernels): out(b), in(b) of the middle vertices, the
wedge-hash tail work per out-degree class.  python scripts/degree_stats.py 22 26"""
import os
import sys
import torch
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from inputs.graphs import rmat_edges_torch, WORKLOADS

dev = "cuda"
for sc in [int(x) for x in sys.argv[1:]]:
    seed = {22: 5, 26: 6, 16: 4}.get(sc, 5)
    n = 1 << sc
    e = rmat_edges_torch(sc, 16, seed, device=dev).to(torch.int64)
    a = torch.minimum(e[:, 0], e[:, 1]); b = torch.maximum(e[:, 0], e[:, 1])
    del e
    ok = a != b
    k = torch.unique(a[ok] * n + b[ok])
    del a, b, ok
    a = k // n; b = k % n
    del k
    m = a.numel()
    deg = torch.bincount(a, minlength=n) + torch.bincount(b, minlength=n)
    key = deg * n + torch.arange(n, device=dev)
    order = torch.argsort(key)
    rank = torch.empty(n, dtype=torch.int64, device=dev)
    rank[order] = torch.arange(n, device=dev)
    u = torch.minimum(rank[a], rank[b]); v = torch.maximum(rank[a], rank[b])
    del a, b
    out = torch.bincount(u, minlength=n); inn = torch.bincount(v, minlength=n)
    print(f"RMAT-{sc}: n {n} m {m} maxdeg {int(deg.max())} max out {int(out.max())}", flush=True)
    s = torch.argsort(u * n + v)
    u = u[s]; v = v[s]
    del s
    oofs = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    oofs[1:] = torch.cumsum(out, 0)
    pos = torch.arange(m, device=dev) - oofs[u]
    tail = out[u] - pos - 1
    ov = out[v]
    print(f"  total tail work {float(tail.sum()):.3e}  merge work all {float((out[u] + ov).sum()):.3e}")
    for lo, hi in [(0, 256), (256, 1024), (1024, 2048), (2048, 4096), (4096, 8192), (8192, 16384), (16384, 1 << 30)]:
        sel = (ov > lo) & (ov <= hi)
        mids = ((out > lo) & (out <= hi) & (inn > 0))
        print(f"  out(b) in ({lo},{hi}]: middles {int(mids.sum())} in-edges {int(sel.sum())} "
              f"tail work {float(tail[sel].sum()):.3e} merge work {float((out[u] + ov)[sel].sum()):.3e} "
              f"max in {int(inn[mids].max()) if mids.any() else 0} min range {int((n - 1 - torch.nonzero(mids).flatten()).min()) if mids.any() else 0} "
              f"max range {int((n - 1 - torch.nonzero(mids).flatten()).max()) if mids.any() else 0}", flush=True)
    del u, v, tail, ov, pos, oofs, out, inn, deg, rank, order, key
    torch.cuda.empty_cache()
