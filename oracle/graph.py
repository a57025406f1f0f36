"""Oracle: the input graph, by definition.  (Test infrastructure only.)

PAPER.md Sec. 2/5: SGC on an undirected graph, edge-induced embeddings.  An
edge list is turned into a simple undirected graph: self loops dropped,
duplicate / reversed duplicates merged (north_star: "edge list ->
deduplicated, symmetrised, degree-ordered CSR").

Degree order (reading R2 in DESIGN.md): new vertex id = position of the vertex
in the list of all vertices sorted by (degree ascending, original id
ascending); each adjacency list is sorted by new id.  This is what the paper's
Sec. 3.6 "degree filtering" / symmetry breaking by "unique vertex ID" (Sec. 3.1)
compare against.
"""
import numpy as np


def simple_adjacency(n, edges):
    """list of Python sets: adj[v] = neighbours of v (no loops, no duplicates)."""
    adj = [set() for _ in range(n)]
    for a, b in edges:
        a = int(a); b = int(b)
        if a != b:
            adj[a].add(b)
            adj[b].add(a)
    return adj


def degree_ordered_csr(n, edges):
    """Definition of the degree-ordered CSR (numpy, straightforward).

    Returns (offsets int64[n+1], adjacency int32[2m], order int64[n]) where
    order[new_id] = original id.
    """
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    e = e[e[:, 0] != e[:, 1]]
    both = np.concatenate([e, e[:, ::-1]], axis=0)
    keys = np.unique(both[:, 0] * n + both[:, 1])          # dedup directed pairs
    src = keys // n
    dst = keys % n
    deg = np.bincount(src, minlength=n).astype(np.int64)
    order = np.lexsort((np.arange(n), deg))                  # by (deg, id)
    rank = np.empty(n, dtype=np.int64)
    rank[order] = np.arange(n)
    ns, nd = rank[src], rank[dst]
    idx = np.lexsort((nd, ns))                                # sort by (src, dst)
    ns, nd = ns[idx], nd[idx]
    offs = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(ns, minlength=n), out=offs[1:])
    return offs, nd.astype(np.int32), order


def csr_to_adjacency(offs, adj):
    """list of Python sets from a CSR."""
    n = len(offs) - 1
    return [set(adj[offs[v]:offs[v + 1]].tolist()) for v in range(n)]
