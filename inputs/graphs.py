"""Synthetic graph generators (raw undirected edge lists).

All generators are seeded and counter-based so the same (seed, size) gives the
same edges on every machine.  They return raw edge lists; turning them into a
deduplicated, symmetrised, degree-ordered CSR is the job of the code under
test (``fsgc_load_graph``) and of the oracle, not of this module.

Workload shapes follow BASELINE.json ``configs`` and PAPER.md Table 1 (Sec. 5):
  * ``pl2k``      2,000 vertices / 10,000 edges power-law (configs[0])
  * ``internet``  124,651 vertices / 193,620 edges, d_avg 3.1, d_max ~151,
                  shaped like Table 1's "internet" row (configs[1])
  * ``rmat22``    RMAT scale 22, edge factor 16 (configs[2]; Table 1 lists
                  rmat16.sym and kron_g500-logn20 as the RMAT/Kronecker inputs)
  * ``pl10m``     power-law, ~10M edges, d_max ~2.5k (configs[3]; d_max chosen so
                  the Fig. 4 count stays below 2^128 -- DESIGN.md R11)
  * ``rmat16``    RMAT scale 16, edge factor 8 (Table 1's rmat16.sym scale)
  * ``rmat26``    RMAT scale 26, edge factor 16, ~1B edges (configs[4])
"""
import os
import numpy as np

from .rng import counter_u64_np, counter_u64_torch

_HERE = os.path.dirname(os.path.abspath(__file__))
_REPO = os.path.dirname(_HERE)


def fig2_edges():
    """(n, edges[m,2] int64) of the PAPER.md Fig. 2 example (tests/golden)."""
    path = os.path.join(_REPO, "tests", "golden", "fig2_graph.txt")
    rows = [ln.split() for ln in open(path) if ln.strip() and not ln.startswith("#")]
    n, m = int(rows[0][0]), int(rows[0][1])
    e = np.array([[int(a), int(b)] for a, b in rows[1:]], dtype=np.int64)
    assert e.shape == (m, 2)
    return n, e


# ---------------------------------------------------------------- power law

def _chung_lu_cdf(n, m, exponent, dmax):
    """Integer CDF (int64, total 2**40) of Chung-Lu endpoint weights
    w_i = (i + i0)^(-1/(exponent-1)), with i0 chosen so the expected degree of
    vertex 0, 2 m w_0 / W, equals ``dmax``."""
    alpha = 1.0 / (exponent - 1.0)
    idx = np.arange(n, dtype=np.float64)

    def top(i0):
        w = (idx + i0) ** (-alpha)
        return 2.0 * m * w[0] / w.sum()

    lo, hi = 1e-6, float(n)
    for _ in range(200):  # top() is decreasing in i0
        mid = (lo * hi) ** 0.5
        if top(mid) > dmax:
            lo = mid
        else:
            hi = mid
    w = (idx + hi) ** (-alpha)
    w = w / w.sum()
    cdf = np.floor(np.cumsum(w) * float(1 << 40)).astype(np.int64)
    cdf[-1] = 1 << 40
    return cdf


def powerlaw_edges(n, m, exponent=2.1, dmax=151, seed=1):
    """Exactly ``m`` distinct undirected non-loop edges, Chung-Lu power law.

    Candidate edge j draws both endpoints from the weight CDF with the 64-bit
    counter value j of stream 11 (high 40 bits -> endpoint a) and stream 12
    (-> endpoint b).  Self loops are skipped, and the first ``m`` distinct
    pairs in candidate order are kept (so the set is reproducible).
    """
    cdf = _chung_lu_cdf(n, m, exponent, dmax)
    keys_out = np.empty(0, dtype=np.int64)
    seen = np.empty(0, dtype=np.int64)
    start = 0
    batch = max(1024, int(m * 1.5))
    while keys_out.size < m:
        ua = (counter_u64_np(seed, 11, start, batch) >> np.uint64(24)).astype(np.int64)
        ub = (counter_u64_np(seed, 12, start, batch) >> np.uint64(24)).astype(np.int64)
        a = np.searchsorted(cdf, ua, side="right")
        b = np.searchsorted(cdf, ub, side="right")
        ok = a != b
        lo = np.minimum(a, b)[ok]
        hi = np.maximum(a, b)[ok]
        keys = lo * n + hi
        uk, first = np.unique(keys, return_index=True)
        fresh = ~np.isin(uk, seen)
        uk, first = uk[fresh], first[fresh]
        uk = uk[np.argsort(first, kind="stable")]
        need = m - keys_out.size
        keys_out = np.concatenate([keys_out, uk[:need]])
        seen = np.sort(keys_out)
        start += batch
    e = np.stack([keys_out // n, keys_out % n], axis=1).astype(np.int64)
    return e


# -------------------------------------------------------------------- RMAT

def _rmat_thresholds(a, b, c):
    ta = int(round(a * 65536))
    tab = int(round((a + b) * 65536))
    tabc = int(round((a + b + c) * 65536))
    return ta, tab, tabc


def rmat_edges_np(scale, edge_factor=16, seed=7, a=0.57, b=0.19, c=0.19,
                  start=0, count=None):
    """RMAT edges [start, start+count) of the (edge_factor << scale) list.

    Level l (0 = most significant bit) of edge e uses the 16-bit slice
    (l % 4) of counter value e of stream 100 + l // 4; quadrant thresholds are
    a, a+b, a+b+c quantised to 1/65536.  Raw list: may contain duplicates and
    self loops (``fsgc_load_graph`` removes them)."""
    total = edge_factor << scale
    if count is None:
        count = total - start
    ta, tab, tabc = _rmat_thresholds(a, b, c)
    src = np.zeros(count, dtype=np.int64)
    dst = np.zeros(count, dtype=np.int64)
    h = None
    for lvl in range(scale):
        if lvl % 4 == 0:
            h = counter_u64_np(seed, 100 + lvl // 4, start, count)
        r = ((h >> np.uint64(16 * (lvl % 4))) & np.uint64(0xFFFF)).astype(np.int64)
        bit = np.int64(1) << np.int64(scale - 1 - lvl)
        row = r >= tab
        col = ((r >= ta) & (r < tab)) | (r >= tabc)
        src |= np.where(row, bit, 0)
        dst |= np.where(col, bit, 0)
    return np.stack([src, dst], axis=1)


def rmat_edges_torch(scale, edge_factor=16, seed=7, a=0.57, b=0.19, c=0.19,
                     start=0, count=None, device="cpu", chunk=1 << 25):
    """Same edges as ``rmat_edges_np`` as an int32 [count, 2] torch tensor,
    generated chunk by chunk on ``device`` (used for scale 22 / 26)."""
    import torch
    total = edge_factor << scale
    if count is None:
        count = total - start
    ta, tab, tabc = _rmat_thresholds(a, b, c)
    out = torch.empty((count, 2), dtype=torch.int32, device=device)
    for off in range(0, count, chunk):
        cnt = min(chunk, count - off)
        src = torch.zeros(cnt, dtype=torch.int64, device=device)
        dst = torch.zeros(cnt, dtype=torch.int64, device=device)
        h = None
        for lvl in range(scale):
            if lvl % 4 == 0:
                h = counter_u64_torch(seed, 100 + lvl // 4, start + off, cnt, device)
            r = (h >> (16 * (lvl % 4))) & 0xFFFF
            bit = 1 << (scale - 1 - lvl)
            row = r >= tab
            col = ((r >= ta) & (r < tab)) | (r >= tabc)
            src |= row.to(torch.int64) * bit
            dst |= col.to(torch.int64) * bit
            del r, row, col
        out[off:off + cnt, 0] = src.to(torch.int32)
        out[off:off + cnt, 1] = dst.to(torch.int32)
        del src, dst, h
    return out


# --------------------------------------------------------------- workloads

WORKLOADS = {
    # name: (kind, params)
    "fig2": ("fig2", {}),
    "pl2k": ("powerlaw", dict(n=2000, m=10000, exponent=2.5, dmax=120, seed=1)),
    "internet": ("powerlaw", dict(n=124651, m=193620, exponent=2.1, dmax=151, seed=2)),
    "pl10m": ("powerlaw", dict(n=1 << 20, m=10_000_000, exponent=2.2, dmax=2500, seed=3)),
    "rmat16": ("rmat", dict(scale=16, edge_factor=8, seed=4)),
    "rmat22": ("rmat", dict(scale=22, edge_factor=16, seed=5)),
    "rmat26": ("rmat", dict(scale=26, edge_factor=16, seed=6)),
}


def workload_edges(name, device=None):
    """(n, edges) for a named workload.  ``device`` selects torch generation
    for RMAT (returns an int32 torch tensor on that device); otherwise numpy
    int64 [m, 2]."""
    kind, p = WORKLOADS[name]
    if kind == "fig2":
        return fig2_edges()
    if kind == "powerlaw":
        return p["n"], powerlaw_edges(**p)
    if kind == "rmat":
        n = 1 << p["scale"]
        if device is not None:
            return n, rmat_edges_torch(p["scale"], p["edge_factor"], p["seed"], device=device)
        return n, rmat_edges_np(p["scale"], p["edge_factor"], p["seed"])
    raise KeyError(name)
