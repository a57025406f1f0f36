"""Oracle, mode 2 in plain C (test infrastructure only, NOT part of the product).

``fringe_count_c`` / ``root_raw_sum_c`` compute exactly what
``oracle.count.fringe_count`` / ``root_raw_sum`` compute -- every injective
core map (no symmetry breaking), the Venn diagram of the anchors' external
neighbour sets by explicit marking (Sec. 3.3-3.4), Listing 5 (Fig. 5)
per map, times prod k_t!, divided by |Aut(P)| (Sec. 3.1) -- with the
per-map work in ``oracle/c/core_fringe.c`` (exact: checked 128-bit fc, 256-bit
sum) so the oracle reaches graphs with real hubs (RMAT scale 10-14) in
seconds.  The decomposition, the search order and the final scaling are the
pinned Python oracle's own (``oracle.pattern``); only the inner loops moved.

Pinned in tests/test_oracle.py against the Python oracle (every connected
pattern <= 5 vertices on random graphs, the named patterns, per-root sums) and
against closed forms at sizes the Python oracle does not reach (k-tailed
triangles = sum over triangles of C(deg - 2, k), k-stars, triangles by
trace(A^3) / 6).

The shared library is built by ``build()`` below (gcc -O2 -fopenmp), called
lazily on first use and by ``__graft_entry__.build()``.
"""
import ctypes as C
import os
import subprocess
from math import factorial

import numpy as np

from .pattern import automorphism_count, decompose, pattern_adjacency

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "c", "core_fringe.c")
_LIB = os.path.join(_HERE, "c", "liboracle.so")
_lib = None


def build(force=False):
    """Compile oracle/c/core_fringe.c -> oracle/c/liboracle.so (gcc)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_SRC) > os.path.getmtime(_LIB):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.run(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC], check=True)
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = C.CDLL(build())
        f = lib.oracle_core_fringe
        f.restype = C.c_int
        f.argtypes = [C.c_int64, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p, C.c_int, C.c_void_p, C.c_int,
                      C.c_void_p, C.c_void_p, C.c_void_p, C.c_int64, C.c_int, C.c_void_p, C.c_void_p,
                      C.c_void_p]
        _lib = lib
    return _lib


def simple_csr(n, edges):
    """The simple undirected graph of an edge list as a CSR with sorted
    adjacency lists, ORIGINAL vertex ids (loops dropped, duplicates merged)."""
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    e = e[e[:, 0] != e[:, 1]]
    both = np.concatenate([e, e[:, ::-1]], axis=0)
    keys = np.unique(both[:, 0] * n + both[:, 1])
    src = keys // n
    offs = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(src, minlength=n), out=offs[1:])
    return offs, (keys % n).astype(np.int32)


def _core_search(n, edges, dec, first=None):
    """the core's search order (BFS from ``first``, neighbours ascending --
    the order of oracle.count._core_homs) and each position's back-adjacency"""
    padj = pattern_adjacency(n, edges)
    cs = sorted(dec.core)
    cset = set(cs)
    first = cs[0] if first is None else first
    order, seen = [first], {first}
    i = 0
    while i < len(order):
        for y in sorted(padj[order[i]] & cset):
            if y not in seen:
                seen.add(y)
                order.append(y)
        i += 1
    pos = {v: k for k, v in enumerate(order)}
    back = [sum(1 << pos[u] for u in padj[v] & cset if pos[u] < k) for k, v in enumerate(order)]
    return order, pos, back


def _run(csr, n_p, edges_p, core, first=None, roots=None, threads=None):
    offs, adj = csr
    dec = decompose(n_p, edges_p, core)
    order, pos, back = _core_search(n_p, edges_p, dec, first)
    bit = {a: j for j, a in enumerate(dec.anchors)}
    anchor_pos = np.array([pos[a] for a in dec.anchors] or [0], dtype=np.int32)
    tanch = np.array([sum(1 << bit[a] for a in A) for A, _ in dec.types] or [0], dtype=np.uint32)
    tk = np.array([kk for _, kk in dec.types] or [0], dtype=np.int32)
    backa = np.array(back, dtype=np.uint32)
    rts = None if roots is None else np.ascontiguousarray(np.asarray(roots, dtype=np.int32))
    raw = np.zeros(4, dtype=np.uint64)
    matches = C.c_int64()
    ovf = C.c_int32()
    nthreads = threads or os.cpu_count() or 1
    rc = _load().oracle_core_fringe(
        len(offs) - 1, offs.ctypes.data, adj.ctypes.data, len(order), backa.ctypes.data, dec.q,
        anchor_pos.ctypes.data, len(dec.types), tanch.ctypes.data, tk.ctypes.data,
        None if rts is None else rts.ctypes.data, 0 if rts is None else len(rts), nthreads,
        raw.ctypes.data, C.byref(matches), C.byref(ovf))
    assert rc == 0
    total = sum(int(raw[i]) << (64 * i) for i in range(4))
    return dec, total, matches.value, bool(ovf.value)


def fringe_count_c(csr, n_p, edges_p, core=None, threads=None):
    """Mode 2 on the whole graph: (count, raw, core maps).  ``csr`` =
    simple_csr(n, edges).  Raises if an fc value exceeds 128 bits."""
    dec, raw, maps, ovf = _run(csr, n_p, edges_p, core, threads=threads)
    if ovf:
        raise OverflowError("an fc value exceeds 2^128 - 1")
    scale = 1
    for _, kk in dec.types:
        scale *= factorial(kk)
    aut = automorphism_count(n_p, edges_p)
    assert (raw * scale) % aut == 0
    return raw * scale // aut, raw, maps


def root_raw_sum_c(csr, n_p, edges_p, core, root_pv, roots, threads=None):
    """sum over roots r of oracle.count.root_raw_sum(..., root_pv, r)"""
    _, raw, maps, ovf = _run(csr, n_p, edges_p, core, first=root_pv, roots=roots, threads=threads)
    if ovf:
        raise OverflowError("an fc value exceeds 2^128 - 1")
    return raw, maps
