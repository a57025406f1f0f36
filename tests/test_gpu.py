"""GPU parity tests (``-m gpu``): the CUDA path, called through the C ABI,
against the oracle on the same seeded inputs.  Integer results: bit-exact.

Expected values come only from ``oracle/`` (or the paper, for Fig. 2).
"""
import os
import random
from math import comb

import numpy as np
import pytest

import oracle
from inputs import PATTERNS, fig2_edges, workload_edges, rmat_edges_np
from inputs.patterns import all_connected_patterns, star

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sc_bradleyab25_b200 as F  # noqa: E402


def oracle_graph(n, edges):
    offs, adj, order = oracle.degree_ordered_csr(n, edges)
    return offs, adj, order, oracle.csr_to_adjacency(offs, adj)


def count_all(g, pats, **kw):
    out = []
    for i in range(0, len(pats), 16):
        out += F.fsgc_count(g, pats[i:i + 16], **kw)
    return out


_cache = {}


# the support pass's two algorithms: the merge kernel (graphs below 2^20
# edges by default) and the wedge-hash kernels (every larger graph: configs[2],
# [3], [4]) -- FSGC_SUP_HASH_MIN_M is read at every fsgc_load_graph
# "block-tables": the listing kernels with the warp-table cap lowered to 4, so
# every middle vertex with out(b) > 4 takes the block-table kernels (on the
# bench graphs those are the heavy middles, out(b) up to 3,004 at RMAT-26)
SUP_MODES = {"merge": {"FSGC_SUP_HASH_MIN_M": str(1 << 40)},
             "wedge-hash": {"FSGC_SUP_HASH_MIN_M": "0"},
             "block-tables": {"FSGC_SUP_HASH_MIN_M": "0", "FSGC_SUP_CAPW": "4"}}


@pytest.fixture(params=sorted(SUP_MODES))
def sup_mode(request, monkeypatch):
    for k, v in SUP_MODES[request.param].items():
        monkeypatch.setenv(k, v)
    return request.param


_ofc_cache = {}


def oracle_fc(key, gadj, P):
    """oracle.fringe_count, memoised per (graph key, pattern) across the
    support-mode parametrisations"""
    k = (key, P.name, P.core)
    if k not in _ofc_cache:
        _ofc_cache[k] = oracle.fringe_count(gadj, P.n, P.edges, P.core)
    return _ofc_cache[k]


def workload(name):
    if name not in _cache:
        n, e = workload_edges(name)
        _cache[name] = (n, e, oracle_graph(n, e))
    return _cache[name]


# ------------------------------------------------------------ graph loading

def _rand_multigraph(n, E, seed):
    rng = np.random.default_rng(seed)
    return rng.integers(0, n, size=(E, 2))


@pytest.mark.parametrize("case", ["fig2", "pl2k", "multi", "rmat10", "isolated", "empty", "int32", "device"])
def test_load_graph_bit_exact(case):
    if case == "fig2":
        n, e = fig2_edges()
    elif case == "pl2k":
        n, e, _ = workload("pl2k")
    elif case == "multi":
        n, e = 300, _rand_multigraph(300, 5000, 1)          # duplicates + loops
    elif case == "rmat10":
        n, e = 1 << 10, rmat_edges_np(10, 8, seed=2)
    elif case == "isolated":
        n, e = 1000, _rand_multigraph(50, 400, 3)           # vertices 50..999 isolated
    elif case == "empty":
        n, e = 7, np.zeros((0, 2), dtype=np.int64)
    elif case == "int32":
        n, e = 500, _rand_multigraph(500, 3000, 4).astype(np.int32)
    else:
        n, e = 800, _rand_multigraph(800, 6000, 5)
    src = torch.from_numpy(np.ascontiguousarray(e)).cuda() if case == "device" else e
    g = F.fsgc_load_graph(src, n)
    offs, adj, order = g.download()
    eo, ea, eord = oracle.degree_ordered_csr(n, e)
    assert np.array_equal(offs, eo)
    assert np.array_equal(adj, ea)
    assert np.array_equal(order, eord)
    assert g.m == len(ea) // 2
    assert g.max_degree == (int(np.diff(eo).max()) if n else 0)


def test_load_graph_rejects_bad_ids():
    with pytest.raises(F.FsgcError):
        F.fsgc_load_graph(np.array([[0, 1], [1, 5]]), 5)
    with pytest.raises(F.FsgcError):
        F.fsgc_load_graph(np.array([[0, -1]]), 5)


# ------------------------------------------------------------ counts

def test_fig2_paper_values():
    """Sec. 1: 1 triangle, 5 tailed triangles; Sec. 3: 35 3-stars."""
    n, e = fig2_edges()
    g = F.fsgc_load_graph(e, n)
    pats = [F.compile_named(PATTERNS[x]) for x in ("triangle", "1-tailed-triangle", "3-star")]
    res = F.fsgc_count(g, pats)
    assert [r.count for r in res] == [1, 5, 35]


@pytest.mark.parametrize("seed", range(3))
def test_all_small_patterns_random_graphs(seed, sup_mode):
    """All 31 connected patterns <= 5 vertices on random graphs vs mode-1
    brute force (Sec. 3.4's exhaustive check, on the GPU path)."""
    rng = random.Random(seed)
    n = 12 + 3 * seed
    edges = [(a, b) for a in range(n) for b in range(a + 1, n) if rng.random() < 0.35]
    g = F.fsgc_load_graph(np.array(edges, dtype=np.int64).reshape(-1, 2), n)
    _, _, _, gadj = oracle_graph(n, edges)
    pats = all_connected_patterns(5)
    res = count_all(g, [F.compile_named(P) for P in pats])
    for P, r in zip(pats, res):
        assert not r.overflow
        assert r.count == oracle.brute_force_count(gadj, P.n, P.edges), P


PL2K_PATTERNS = ["1-tailed-triangle", "2-tailed-triangle", "3-tailed-triangle", "4-tailed-triangle",
                 "triangle", "wedge", "3-star", "6-star", "path4", "path5", "cycle4", "clique4",
                 "diamond", "fig4", "k4core+2f", "k4core+6f", "diamondcore+3f", "tricore+4f",
                 "tricore+6f", "c4core+2f", "clique5", "cycle5"]


def test_pl2k_named_patterns(sup_mode):
    """configs[0] graph (2,000 vertices / 10,000 edges) -- every named pattern
    vs the oracle's core+fringe mode (itself pinned to brute force)."""
    n, e, (_, _, _, gadj) = workload("pl2k")
    g = F.fsgc_load_graph(e, n)
    pats = [PATTERNS[x] for x in PL2K_PATTERNS]
    res = count_all(g, [F.compile_named(P) for P in pats])
    for P, r in zip(pats, res):
        want = oracle_fc("pl2k", gadj, P)
        assert not r.overflow and r.count == want, (P.name, r.count, want)


def test_symmetry_breaking_invariant():
    """sum over symmetry-broken core instances x fringe programs == sum over
    all injective core maps (divided consistently)."""
    n, e, _ = workload("pl2k")
    g = F.fsgc_load_graph(e, n)
    pats = [F.compile_named(PATTERNS[x]) for x in ["1-tailed-triangle", "cycle4", "clique4", "diamond",
                                                     "fig4", "k4core+3f", "diamondcore+2f", "c4core+4f"]]
    a = count_all(g, pats)
    b = count_all(g, pats, no_symmetry_breaking=True)
    for x, y in zip(a, b):
        assert x.count == y.count and x.count is not None


def test_batch_equals_single_and_shards_partition():
    n, e, _ = workload("internet")
    g = F.fsgc_load_graph(e, n)
    pats = [F.compile_named(PATTERNS[f"{k}-tailed-triangle"]) for k in range(1, 5)]
    batch = F.fsgc_count(g, pats)
    for p, r in zip(pats, batch):
        assert F.fsgc_count(g, [p])[0].count == r.count
    for shards in (2, 3, 8):
        raws = [0] * 4
        for s in range(shards):
            part = F.fsgc_count(g, pats, shard_index=s, shard_count=shards)
            for k in range(4):
                raws[k] += part[k].raw
        assert raws == [r.raw for r in batch]


def test_internet_full_size_bench_config(sup_mode):
    """configs[1] at full size, in the launch configuration bench.py times
    (one batched pass over the 4 k-tailed triangles): every count exact."""
    n, e, (_, _, _, gadj) = workload("internet")
    g = F.fsgc_load_graph(e, n)
    pats = [PATTERNS[f"{k}-tailed-triangle"] for k in range(1, 5)]
    res = F.fsgc_count(g, [F.compile_named(P) for P in pats])
    for P, r in zip(pats, res):
        assert r.count == oracle_fc("internet", gadj, P), P.name


@pytest.mark.parametrize("wl", ["internet", "rmat16"])
def test_sampled_roots_no_symmetry(wl):
    """Per-root-vertex raw sums (no symmetry breaking) for sampled roots,
    low and high degree, vs oracle.root_raw_sum."""
    n, e, (offs, _, _, gadj) = workload(wl)
    g = F.fsgc_load_graph(e, n)
    rng = random.Random(3)
    deg = np.diff(offs)
    if wl == "internet":   # d_max ~170: the hubs themselves are cheap for the oracle
        cands = [n - 1 - i for i in range(5)] + rng.sample(range(n), 10)
    else:                  # RMAT hubs are too heavy for a per-root Python oracle
        ok = [v for v in range(n) if 1 <= deg[v] <= 48]
        cands = rng.sample(ok, 10) + [ok[-1]]
    names = ["1-tailed-triangle", "4-tailed-triangle", "diamond", "tricore+3f"] if wl == "internet" \
        else ["1-tailed-triangle", "cycle4", "diamond", "k4core+2f"]
    for name in names:
        P = PATTERNS[name]
        p = F.compile_named(P)
        for r in cands:
            if p.info.core_size == 1:
                b, e_ = r, r + 1
            else:
                b, e_ = int(offs[r]), int(offs[r + 1])
            res = F.fsgc_count(g, [p], root_begin=b, root_end=e_, no_symmetry_breaking=True)[0]
            want = oracle.root_raw_sum(gadj, P.n, P.edges, P.core, res.root_pattern_vertex, r)
            assert res.raw == want, (name, r, res.raw, want)


def test_overflow_and_192bit_binomials():
    """Star graph with 200,000 leaves: C(200000, 8) < 2^128 but 8*C(n,8) >
    2^128 (exercises the 192-bit intermediate); C(200000, 9) > 2^128 must be
    flagged, never wrapped."""
    L = 200000
    e = np.stack([np.zeros(L, dtype=np.int64), np.arange(1, L + 1)], axis=1)
    g = F.fsgc_load_graph(e, L + 1)
    r7, r8, r9 = F.fsgc_count(g, [F.compile_named(star(k)) for k in (7, 8, 9)])
    assert r7.count == comb(L, 7) and r8.count == comb(L, 8)
    assert comb(L, 8) < 1 << 128 < 8 * comb(L, 8)
    assert r9.overflow and r9.count is None and comb(L, 9) >= 1 << 128


def test_degenerate_inputs():
    g = F.fsgc_load_graph(np.zeros((0, 2), dtype=np.int64), 5)
    res = F.fsgc_count(g, [F.compile_named(PATTERNS[x]) for x in ("vertex", "edge", "triangle", "3-star")])
    assert [r.count for r in res] == [5, 0, 0, 0]
    n, e = fig2_edges()
    g = F.fsgc_load_graph(e, n)
    big = F.compile_named(PATTERNS["clique5"])
    assert F.fsgc_count(g, [big])[0].count == 0
    r = F.fsgc_count(g, [F.compile_named(PATTERNS["edge"])], root_begin=3, root_end=3)[0]
    assert r.raw == 0
    assert F.fsgc_count(g, [F.compile_named(PATTERNS["vertex"]), F.compile_named(PATTERNS["edge"])]) [1].count == 8


def test_degree_filter_off_counts_core_instances():
    n, e, (_, _, _, gadj) = workload("pl2k")
    g = F.fsgc_load_graph(e, n)
    for name in ["1-tailed-triangle", "clique4", "cycle4"]:
        P = PATTERNS[name]
        r = F.fsgc_count(g, [F.compile_named(P)], no_degree_filter=True)[0]
        assert r.core_matches == oracle.core_matches(gadj, P.n, P.edges, P.core), name
        assert r.count == F.fsgc_count(g, [F.compile_named(P)])[0].count


def _hub_graph(seed, n=1500, hubs=6, p_hub=0.2, p=0.004):
    rng = np.random.default_rng(seed)
    e = [(a, b) for a in range(hubs) for b in range(a + 1, hubs)]
    for h in range(hubs):
        nb = np.nonzero(rng.random(n) < p_hub)[0]
        e += [(h, int(x)) for x in nb if x != h]
    m = int(p * n * n / 2)
    e += [tuple(x) for x in rng.integers(0, n, size=(m, 2)).tolist()]
    return n, np.array(e, dtype=np.int64)


def test_triangle_core_kernel_with_hub_bitmaps(monkeypatch):
    """Triangle-core fast path (hub bitmaps + warp-cooperative triple
    intersections for heavy roots) vs the oracle, and bitmaps on == off."""
    n, e = _hub_graph(4)
    _, _, _, gadj = oracle_graph(n, e)
    names = ["clique4", "tricore+3f", "tricore+6f", "fig4"]
    pats = [PATTERNS[x] for x in names]
    g_hub = F.fsgc_load_graph(e, n)
    monkeypatch.setenv("FSGC_HUB_BYTES", "0")
    g_nohub = F.fsgc_load_graph(e, n)
    monkeypatch.delenv("FSGC_HUB_BYTES")
    assert g_hub.info.num_vertices == n
    cps = [F.compile_named(P) for P in pats]
    a = F.fsgc_count(g_hub, cps)
    b = F.fsgc_count(g_nohub, cps)
    c = F.fsgc_count(g_hub, cps, no_symmetry_breaking=True)   # generic kernel
    for P, x, y, z in zip(pats, a, b, c):
        assert x.count == y.count == z.count, P.name
    for P, x in zip(pats[:2], a[:2]):
        assert x.count == oracle.fringe_count(gadj, P.n, P.edges, P.core), P.name


def _edge_core_pattern(k, l, m):
    """edge core {0,1}: k tails on 0, l tails on 1, m wedge fringes (Sec. 3.1)."""
    from inputs.patterns import _p
    e = [(0, 1)]
    nxt = 2
    for _ in range(k):
        e.append((0, nxt)); nxt += 1
    for _ in range(l):
        e.append((1, nxt)); nxt += 1
    for _ in range(m):
        e += [(0, nxt), (1, nxt)]; nxt += 1
    return _p(f"edge+{k}t{l}t{m}w", nxt, e)


def test_edge_core_counts_beyond_64_bits():
    """Two adjacent hubs with 1,200 / 1,000 private leaves and 20 common
    neighbours: edge-core counts with up to 12 fringes exceed 2^64.  The bench
    kernel's three arithmetic tiers all run: 64-bit term table (leaf edges),
    128-bit term table (N^K < 2^127), checked per-program 128-bit (12
    fringes, N ~ 2^11: N^K > 2^127).  vs the oracle."""
    A, B = 0, 1
    e = [(A, B)]
    nxt = 2
    for _ in range(1200):
        e.append((A, nxt)); nxt += 1
    for _ in range(1000):
        e.append((B, nxt)); nxt += 1
    for _ in range(20):
        e += [(A, nxt), (B, nxt)]; nxt += 1
    for i in range(2, 200, 2):                        # a few leaf-leaf edges
        e.append((i, i + 1))
    n = nxt
    e = np.array(e, dtype=np.int64)
    _, _, _, gadj = oracle_graph(n, e)
    pats = [_edge_core_pattern(*x) for x in [(6, 4, 0), (8, 0, 1), (3, 3, 3), (5, 5, 0), (1, 0, 1), (2, 1, 2), (7, 4, 1)]]
    g = F.fsgc_load_graph(e, n)
    res = F.fsgc_count(g, [F.compile_named(P) for P in pats])
    assert any(r.count is not None and r.count >= 1 << 64 for r in res)
    for P, r in zip(pats, res):
        assert not r.overflow and r.count == oracle.fringe_count(gadj, P.n, P.edges, P.core), P.name


@pytest.mark.parametrize("algo", ["merge", "wedge-hash", "block-tables"])
def test_sharded_support_stages_sum_to_whole(algo, monkeypatch):
    """FSGC_FLAG_SHARD_SUPPORT: each shard lists its interleaved part of the
    triangles into a partial support array; the SUM of the partial arrays
    (what the multi-GPU all-reduce computes) is the full support array, and
    stage 2 on it gives per-shard raws that sum to the unsharded raw -- for
    an edge-core, a triangle-core and a general-core pass in one plan, with
    either support algorithm (the hash kernels deal their units)."""
    from paper_conf_sc_bradleyab25_b200 import _lib
    for k, v in SUP_MODES[algo].items():
        monkeypatch.setenv(k, v)
    n, e, _ = workload("pl2k")
    g = F.fsgc_load_graph(e, n)
    pats = [F.compile_named(PATTERNS[x]) for x in ["2-tailed-triangle", "tricore+3f", "k4core+2f", "cycle4"]]
    whole = F.fsgc_count(g, pats)
    full = F.Plan(g, pats)
    full.enqueue()
    torch.cuda.synchronize()
    ref_sup = full.support().clone()
    assert int(ref_sup.sum()) > 0
    for shards in (2, 3):
        plans = [F.Plan(g, pats, shard_index=s, shard_count=shards, shard_support=True) for s in range(shards)]
        for P in plans:
            P.enqueue_stage(_lib.FSGC_STAGE_SUPPORT)
        torch.cuda.synchronize()
        tot = sum(P.support().to(torch.int64) for P in plans)
        assert torch.equal(tot.to(torch.int32), ref_sup)
        for P in plans:
            assert not torch.equal(P.support(), ref_sup)      # each part really is partial
            P.support().copy_(tot.to(torch.int32))
            P.enqueue_stage(_lib.FSGC_STAGE_COUNT)
        torch.cuda.synchronize()
        raws = [0] * len(pats)
        for P in plans:
            for k, r in enumerate(P.decode()):
                raws[k] += r.raw
        assert raws == [r.raw for r in whole]
    with pytest.raises(F.FsgcError):
        F.fsgc_count(g, pats, shard_index=0, shard_count=2, shard_support=True)
    with pytest.raises(F.FsgcError):
        F.Plan(g, pats, shard_index=0, shard_count=2, shard_support=True).enqueue()


def _dist_worker(rank, world, port, q):
    import os
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, e = workload_edges("pl2k")
    g = F.fsgc_load_graph(e, n)
    names = ["1-tailed-triangle", "tricore+2f", "diamond", "3-star"]
    pats = [F.compile_named(PATTERNS[x]) for x in names]
    res = F.fsgc_count_distributed(g, pats)
    if rank == 0:
        q.put([r.count for r in res])
    dist.barrier()
    dist.destroy_process_group()


def test_count_distributed_two_ranks_gloo_on_one_gpu():
    """fsgc_count_distributed end to end with 2 ranks (gloo over CUDA tensors,
    both on cuda:0): sharded support + all-reduce, sharded roots + the
    128-bit all-reduce == the single-process count."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + random.Random().randint(0, 2000)
    procs = [ctx.Process(target=_dist_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    n, e, _ = workload("pl2k")
    g = F.fsgc_load_graph(e, n)
    names = ["1-tailed-triangle", "tricore+2f", "diamond", "3-star"]
    want = [r.count for r in F.fsgc_count(g, [F.compile_named(PATTERNS[x]) for x in names])]
    assert got == want


def test_venn_term_table_tiers_vs_oracle(sup_mode):
    """Triangle- and 4-clique-core counts through the Venn term table in all
    three arithmetic tiers -- 64-bit (small leaf triangles), 128-bit and the
    checked Listing 5 fallback (the hub triangle: 13 fringes over ~2^11-sized
    regions, bound > 2^119) -- vs the oracle."""
    rng = np.random.default_rng(11)
    A, B, Cc = 0, 1, 2
    e = [(A, B), (A, Cc), (B, Cc)]
    nxt = 3
    for h in (A, B, Cc):
        for _ in range(3000):
            e.append((h, nxt)); nxt += 1
    for _ in range(60):
        e += [(A, nxt), (B, nxt), (Cc, nxt)]; nxt += 1
    for x, y in ((A, B), (A, Cc), (B, Cc)):
        for _ in range(60):
            e += [(x, nxt), (y, nxt)]; nxt += 1
    leaves = np.arange(3, nxt)
    for _ in range(4000):                                  # small triangles among the leaves
        a, b = rng.choice(leaves, 2, replace=False)
        e.append((int(a), int(b)))
    n = nxt
    e = np.array(e, dtype=np.int64)
    _, _, _, gadj = oracle_graph(n, e)
    names = ["fig4", "tricore+6f", "clique4", "k4core+6f"]
    pats = [PATTERNS[x] for x in names]
    g = F.fsgc_load_graph(e, n)
    res = F.fsgc_count(g, [F.compile_named(P) for P in pats])
    assert res[0].count is not None and res[0].count >= 1 << 100
    for P, r in zip(pats, res):
        assert not r.overflow and r.count == oracle_fc("venn-tiers", gadj, P), P.name


def test_k_tailed_triangles_rmat16_closed_form(sup_mode):
    """RMAT-16 (hubs of degree ~6k next to leaf edges): the edge-core pass runs
    its 64- and 128-bit term-table tiers side by side in one block; every
    k-tailed triangle count must equal the closed form sum over triangles of
    C(deg x - 2, k) (oracle.k_tailed_triangles, pinned), in one batch and
    alone, and twice (deterministic)."""
    n, e, (_, _, _, gadj) = workload("rmat16")
    g = F.fsgc_load_graph(e, n)
    ks = [1, 4]
    pats = [F.compile_named(PATTERNS[f"{k}-tailed-triangle"]) for k in range(1, 5)]
    batch = F.fsgc_count(g, pats)
    again = F.fsgc_count(g, pats)
    assert [r.raw for r in batch] == [r.raw for r in again]
    for k in ks:
        key = ("rmat16-ktt", k)
        if key not in _ofc_cache:
            _ofc_cache[key] = oracle.k_tailed_triangles(gadj, k)
        want = _ofc_cache[key]
        assert not batch[k - 1].overflow and batch[k - 1].count == want, k
        assert F.fsgc_count(g, [pats[k - 1]])[0].count == want, k


def test_triangle_core_z_tiers_hub_closed_form(sup_mode):
    """Triangle core forced (configs[4] patterns) on a hub of degree 200k whose
    triangles mix with hub-free ones: the row-free Z-term path evaluates each
    pattern in 64 or 128 bits by the per-pattern threshold on the leaf's
    largest degree (4-tailed: 128-bit for hub leaves, 3-tailed and below:
    64-bit), so both tiers and both tier choices meet in one warp.  Every
    k-tailed triangle/tricore count equals the closed form sum over triangles
    of C(deg x - 2, k) (oracle.k_tailed_triangles, pinned), and the triangle
    count the plain listing."""
    import numpy as np
    rng = np.random.default_rng(11)
    H = 200_000
    hub = np.stack([np.zeros(H, np.int64), np.arange(1, H + 1)], 1)
    leaf = rng.integers(1, 20_001, size=(6000, 2))
    extra = rng.integers(H + 1, H + 3001, size=(20000, 2))   # a hub-free dense-ish part
    e = np.concatenate([hub, leaf, extra])
    n = H + 3001
    offs, adj, _ = oracle.degree_ordered_csr(n, e)
    gadj = oracle.csr_to_adjacency(offs, adj)
    g = F.fsgc_load_graph(e, n)
    names = ["triangle/tricore", "tricore+1f"] + [f"{k}-tailed-triangle/tricore" for k in (2, 3, 4)]
    res = F.fsgc_count(g, [F.compile_named(PATTERNS[x]) for x in names])
    want = [oracle.k_tailed_triangles(gadj, 0) // 3] + [oracle.k_tailed_triangles(gadj, k) for k in (1, 2, 3, 4)]
    for x, r, w in zip(names, res, want):
        assert not r.overflow and r.count == w, (x, r.count, w)


@pytest.mark.parametrize("wl", ["rmat16", "pl2k"])
def test_wedge_hash_support_equals_merge(wl, monkeypatch):
    """The support pass's two algorithms -- the wedge-hash kernels (middle
    vertex tables; forced with FSGC_SUP_HASH_MIN_M=0) and the merge kernel
    (graphs below the threshold) -- give the identical int32[m] support array
    and identical counts (edge, triangle and 4-clique cores)."""
    n, e, _ = workload(wl)
    names = ["2-tailed-triangle", "tricore+3f", "k4core+2f"]
    pats = [F.compile_named(PATTERNS[x]) for x in names]
    out = []
    for mode in ("wedge-hash", "block-tables", "merge"):
        for k in ("FSGC_SUP_HASH_MIN_M", "FSGC_SUP_CAPW"):
            monkeypatch.delenv(k, raising=False)
        for k, v in SUP_MODES[mode].items():
            monkeypatch.setenv(k, v)
        g = F.fsgc_load_graph(e, n)
        plan = F.Plan(g, pats)
        plan.enqueue()
        torch.cuda.synchronize()
        out.append((plan.support().clone(), [r.raw for r in plan.decode()]))
    for o in out[1:]:
        assert torch.equal(out[0][0], o[0])
        assert out[0][1] == o[1]


def _one_count_subprocess(wl, names, env_extra):
    """counts of ``names`` on workload ``wl`` in a fresh process (the library
    reads its FSGC_* knobs once per process)"""
    import ast
    import subprocess
    import sys
    env = dict(os.environ, **env_extra)
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "scripts", "one_count.py"), wl, ",".join(names), "1"],
                         env=env, capture_output=True, text=True, timeout=600, check=True).stdout
    d = ast.literal_eval(out.strip().splitlines()[-1])
    return {k: v[0] for k, v in d.items()}


@pytest.mark.parametrize("knob", ["FSGC_NO_ZONLY", "FSGC_NO_Z_TERMS"])
def test_triangle_core_fc_paths_agree_rmat18(knob):
    """configs[4]'s pattern set on RMAT-18 (hubs of degree ~25k: both the 64-
    and 128-bit tiers of the Z-term path): the Z-only kernels (default), the
    general triangle-core kernels on the Z path (FSGC_NO_ZONLY=1) and the
    Venn-term / Listing 5 path (FSGC_NO_Z_TERMS=1) give identical counts;
    the k-tailed members also equal the edge-core decomposition of the same
    pattern (independent kernels: support pass + Sec. 3.1 closed form)."""
    from inputs.patterns import CONFIG_PATTERNS
    names = CONFIG_PATTERNS["rmat26"]
    base = _one_count_subprocess("rmat18x", names, {})
    other = _one_count_subprocess("rmat18x", names, {knob: "1"})
    assert base == other
    edge = _one_count_subprocess("rmat18x", ["triangle"] + [f"{k}-tailed-triangle" for k in (2, 3, 4)], {})
    assert base["triangle/tricore"] == edge["triangle"]
    for k in (2, 3, 4):
        assert base[f"{k}-tailed-triangle/tricore"] == edge[f"{k}-tailed-triangle"], k


def test_rmat26_full_size_wedge_hash_equals_merge():
    """configs[4] graph at full size (RMAT-26, 1.05e9 distinct edges): the
    triangle and k-tailed-triangle counts of the bench path (wedge-hash
    support pass) equal those of the independent merge-only support pass
    (FSGC_SUP_MERGE_ONLY=1), and the triangle count is below the Turan-type
    bound m^1.5 (property checks at a size the oracle cannot reach)."""
    names = ["triangle", "1-tailed-triangle", "2-tailed-triangle"]
    a = _one_count_subprocess("rmat26", names, {})
    b = _one_count_subprocess("rmat26", names, {"FSGC_SUP_MERGE_ONLY": "1"})
    assert a == b, (a, b)
    assert 0 < a["triangle"] < (1_051_923_859 ** 1.5)


# ------------------------------------------------ hub-heavy RMAT, symmetry broken
# The bench configurations count with symmetry breaking on skewed graphs; the
# full counts of those kernel paths (triangle-core kernel with hubs, general
# core kernel heavy roots / warp paths / hub bitmaps, both support algorithms)
# against the C oracle (oracle/cfast.py: every injective core map, explicit
# Venn, Listing 5; pinned to the Python oracle and closed forms).
_coracle = {}


def _rmat_case(scale):
    from oracle.cfast import simple_csr
    key = ("rmat", scale)
    if key not in _coracle:
        n = 1 << scale
        e = rmat_edges_np(scale, 16, seed=9)
        _coracle[key] = (n, e, simple_csr(n, e))
    return _coracle[key]


def _c_count(scale, P):
    from oracle.cfast import fringe_count_c
    key = (scale, P.name)
    if key not in _coracle:
        n, e, csr = _rmat_case(scale)
        _coracle[key] = fringe_count_c(csr, P.n, P.edges, P.core)[0]
    return _coracle[key]


RMAT_CASES = [
    (12, ["triangle", "1-tailed-triangle", "3-tailed-triangle", "tricore+1f", "tricore+3f", "tricore+6f",
          "triangle/tricore", "tricore+2f", "2-tailed-triangle/tricore", "4-tailed-triangle/tricore",
          "diamond/tricore"]),
    (8, ["fig4"]),
    (9, ["clique4", "k4core+2f", "diamondcore+3f", "cycle4", "c4core+2f", "diamond"]),
]


@pytest.mark.parametrize("case", range(len(RMAT_CASES)))
def test_rmat_hubs_symmetry_broken_vs_c_oracle(case, sup_mode):
    scale, names = RMAT_CASES[case]
    n, e, _ = _rmat_case(scale)
    g = F.fsgc_load_graph(e, n)
    pats = [PATTERNS[x] for x in names]
    res = F.fsgc_count(g, [F.compile_named(P) for P in pats])
    for P, r in zip(pats, res):
        want = _c_count(scale, P)
        assert not r.overflow and r.count == want, (scale, P.name, r.count, want)


def _bench_line(args, nproc=None, extra_env=None):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, **(extra_env or {}))
    if nproc:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
               "--master-addr=127.0.0.1", f"--master-port={29600 + random.Random().randint(0, 2000)}",
               os.path.join(root, "bench.py")] + args
    else:
        cmd = [sys.executable, os.path.join(root, "bench.py")] + args
    out = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=root)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


@pytest.mark.parametrize("wl", ["pl2k", "internet"])
def test_bench_torchrun_two_ranks_equals_one(wl):
    """bench.py under torchrun with 2 ranks (FSGC_BENCH_BACKEND=gloo: both
    ranks share this box's GPU; the product path is NCCL) reports the same
    counts as the single-process run, and the N=2 line is well formed."""
    args = ["--workload", wl, "--steps", "3", "--warmup", "3", "--no-e2e", "--no-cpu-baseline",
            "--no-per-config"]
    one = _bench_line(args + ["--gpus", "1"])
    two = _bench_line(args + ["--gpus", "2"], nproc=2, extra_env={"FSGC_BENCH_BACKEND": "gloo"})
    assert one["config"]["counts"] == two["config"]["counts"]
    assert two["n_gpus"] == 2 and one["n_gpus"] == 1
    assert two["config"]["core_matches_per_step"] == one["config"]["core_matches_per_step"]
