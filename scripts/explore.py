#!/usr/bin/env python
"""Quick exploration on the GPU: load a workload, count each of its patterns
(or the given ones) once, print count, core matches and kernel times.

    python scripts/explore.py rmat22 [pattern ...]
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import paper_conf_sc_bradleyab25_b200 as F  # noqa: E402
from inputs import workload_edges  # noqa: E402
from inputs.patterns import CONFIG_PATTERNS, PATTERNS  # noqa: E402


def main():
    wl = sys.argv[1]
    names = sys.argv[2:] or CONFIG_PATTERNS[wl]
    if os.environ.get("ROOTS"):        # count only a prefix of the root items
        pass
    dev = torch.device("cuda", 0)
    t = time.time()
    if wl.startswith("rmat"):
        n, e = workload_edges(wl, device=dev)
    elif wl.startswith("pl:"):          # pl:n:m:gamma:dmax
        from inputs.graphs import powerlaw_edges
        _, n_, m_, g_, d_ = wl.split(":")
        n, e = int(n_), powerlaw_edges(int(n_), int(m_), float(g_), float(d_), seed=3)
    else:
        n, e = workload_edges(wl)
    torch.cuda.synchronize()
    print(f"[{wl}] generated {len(e)} raw edges in {time.time() - t:.1f}s", flush=True)
    t = time.time()
    g = F.fsgc_load_graph(e, n)
    torch.cuda.synchronize()
    print(f"[{wl}] CSR n={g.n} m={g.m} dmax={g.max_degree} built in {time.time() - t:.2f}s", flush=True)
    for name in names:
        p = F.compile_named(PATTERNS[name])
        t = time.time()
        r = F.fsgc_count(g, [p])[0]
        dt = time.time() - t
        print(f"  {name:22s} core={p.core_order} types={[(sorted(a), k) for a, k in p.types]} "
              f"count={r.count} ovf={r.overflow} matches={r.core_matches} wall={dt:.3f}s "
              f"kernel={r.kernel_ms:.3f}ms aux={r.aux_ms:.3f}ms", flush=True)


if __name__ == "__main__":
    main()
