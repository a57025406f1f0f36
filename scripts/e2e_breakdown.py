#!/usr/bin/env python
"""Host-clock breakdown of the e2e step (load from pinned host edges + count)
on the bench workload: where the time between the device kernels goes.

    python scripts/e2e_breakdown.py [workload]
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import paper_conf_sc_bradleyab25_b200 as F
from inputs import workload_edges
from inputs.patterns import CONFIG_PATTERNS, PATTERNS

wl = sys.argv[1] if len(sys.argv) > 1 else "internet"
n, e = workload_edges(wl)
e_host = torch.from_numpy(np.ascontiguousarray(e.astype(np.int32))).pin_memory()
cps = [F.compile_named(PATTERNS[x]) for x in CONFIG_PATTERNS[wl]]


def t(f, reps=30):
    out = []
    for _ in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = f()
        torch.cuda.synchronize()
        out.append((time.perf_counter() - t0) * 1e3)
    return float(np.median(out)), r


for _ in range(3):
    g = F.fsgc_load_graph(e_host, n)
    F.fsgc_count(g, cps)
    g.free()
ms_load, _ = t(lambda: F.fsgc_load_graph(e_host, n))
g = F.fsgc_load_graph(e_host, n)
F.fsgc_count(g, cps)
ms_count_cached, _ = t(lambda: F.fsgc_count(g, cps))


def fresh():
    g2 = F.fsgc_load_graph(e_host, n)
    t0 = time.perf_counter()
    F.fsgc_count(g2, cps)
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t0) * 1e3
    t1 = time.perf_counter()
    g2.free()
    return dt, (time.perf_counter() - t1) * 1e3


vals = [fresh() for _ in range(20)]
ms_count_new = float(np.median([v[0] for v in vals]))
ms_free = float(np.median([v[1] for v in vals]))
ms_step, _ = t(lambda: (lambda g2: (F.fsgc_count(g2, cps), g2))(F.fsgc_load_graph(e_host, n)))
print(f"{wl}: load {ms_load:.3f} ms | count (cached plan) {ms_count_cached:.3f} ms | "
      f"count (new graph -> new plan) {ms_count_new:.3f} ms | free {ms_free:.3f} ms | "
      f"load+count {ms_step:.3f} ms")
