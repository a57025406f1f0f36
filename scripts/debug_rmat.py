#!/usr/bin/env python
"""Per-pattern timing / sanity sweep over RMAT scales (GPU helper).

    python scripts/debug_rmat.py SCALES PATTERNS [--nofilter]
e.g. python scripts/debug_rmat.py 16,18,20 triangle,diamond,1-tailed-triangle
Each (scale, pattern) runs in this process; errors are printed, not raised.
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

import paper_conf_sc_bradleyab25_b200 as F
from inputs import PATTERNS
from inputs.graphs import rmat_edges_torch

scales = [int(x) for x in sys.argv[1].split(",")]
names = sys.argv[2].split(",")
ef = int(os.environ.get("EF", "16"))
for sc in scales:
    e = rmat_edges_torch(sc, ef, seed=5, device="cuda")
    g = F.fsgc_load_graph(e, 1 << sc)
    del e
    print(f"scale {sc}: n={g.n} m={g.m} dmax={g.max_degree}", flush=True)
    for nm in names:
        p = F.compile_named(PATTERNS[nm])
        for kw in ({}, {"no_degree_filter": True}):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            try:
                r = F.fsgc_count(g, [p], **kw)[0]
                dt = time.perf_counter() - t0
                print(f"  {nm:22s} {str(kw):30s} {dt*1e3:10.2f} ms  count={r.count} raw={r.raw} "
                      f"div={r.divisor} ovf={r.overflow} matches={r.core_matches} kind={r.pass_kind} "
                      f"kms={r.kernel_ms:.2f} ams={r.aux_ms:.2f}", flush=True)
            except Exception as ex:   # noqa: BLE001
                print(f"  {nm:22s} {str(kw):30s} ERROR {ex}", flush=True)
    g.free()
