"""The bench's roofline byte model on small graphs, CPU
only: `listing_stats` (degree-ordered orientation, per-edge tail lengths of
the listing kernels, merge lengths) against a brute-force count written from
the definitions, and the byte formulas' units."""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _brute(n, e):
    """oriented simple graph by (degree, id) order; for every oriented edge
    (a, b): the tail of N+(a) after b and out(a) + out(b)"""
    edges = {(min(a, b), max(a, b)) for a, b in e if a != b}
    deg = [0] * n
    for a, b in edges:
        deg[a] += 1
        deg[b] += 1
    rank = {v: i for i, v in enumerate(sorted(range(n), key=lambda v: (deg[v], v)))}
    out = {}
    for a, b in edges:
        u, v = sorted((rank[a], rank[b]))
        out.setdefault(u, []).append(v)
    tail = merge = 0
    for u, lst in out.items():
        lst.sort()
        for i, v in enumerate(lst):
            tail += len(lst) - i - 1
            merge += len(lst) + len(out.get(v, []))
    return len(edges), tail, merge


@pytest.mark.parametrize("seed", range(3))
def test_listing_stats_matches_definition(seed):
    import bench
    rng = np.random.default_rng(seed)
    n = 60
    e = rng.integers(0, n, size=(400, 2))
    e = np.concatenate([e, np.stack([np.zeros(40, np.int64), np.arange(1, 41)], 1)])   # a hub
    st = bench.listing_stats(n, e)
    m, tail, merge = _brute(n, e.tolist())
    assert st["m"] == m and st["tail"] == tail and st["merge"] == merge


def test_byte_model_formulas():
    import bench
    st = {"m": 10, "tail": 100.0, "merge": 50.0}
    assert bench.support_bytes(st, 7, True) == 44 * 10 + 4 * 100 + 8 * 7
    assert bench.support_bytes(st, 7, False) == 40 * 10 + 4 * 50
    assert bench.tricore_bytes(st, 7) == 76 * 10 + 4 * 100 + 4 * 7
