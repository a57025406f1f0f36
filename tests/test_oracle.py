"""Pins for the oracle (``-m "not gpu"``): the oracle is checked against what
PAPER.md and mathematics fix, never against itself or the CUDA path.

Citations are to PAPER.md sections / equations / listings (the extracted text
is a single line, so line numbers are not meaningful).
"""
import itertools
import random
from math import comb, factorial

import numpy as np
import pytest

import oracle
from inputs import PATTERNS, fig2_edges
from inputs.patterns import all_connected_patterns, star, Pattern


def rand_graph(n, p, seed):
    rng = random.Random(seed)
    edges = [(a, b) for a in range(n) for b in range(a + 1, n) if rng.random() < p]
    return edges, oracle.simple_adjacency(n, edges)


def adjmat(gadj):
    n = len(gadj)
    A = np.zeros((n, n), dtype=np.int64)
    for v in range(n):
        for w in gadj[v]:
            A[v, w] = 1
    return A


# ------------------------------------------------------------ Fig. 2 (golden)

@pytest.mark.parametrize("mode", ["brute", "fringe"])
def test_fig2_worked_example(mode):
    """Sec. 1: "There is only one triangle in this graph (formed by vertices
    0, 1, and 2), but there are five unique tailed triangles."  Sec. 3: vertex
    0 is the centre of binom(7,3) = 35 3-stars and is the only possible one."""
    n, e = fig2_edges()
    g = oracle.simple_adjacency(n, e)
    f = oracle.brute_force_count if mode == "brute" else oracle.fringe_count
    tri, tt, s3 = PATTERNS["triangle"], PATTERNS["1-tailed-triangle"], PATTERNS["3-star"]
    assert f(g, tri.n, tri.edges) == 1
    assert f(g, tt.n, tt.edges) == 5
    assert f(g, s3.n, s3.edges) == 35
    assert len(g[0]) == 7 and all(len(g[v]) < 3 for v in range(1, n))


# ------------------------------------------------------------ closed forms

@pytest.mark.parametrize("seed", range(6))
def test_closed_forms_random(seed):
    n = 14 + seed
    edges, g = rand_graph(n, 0.3, seed)
    A = adjmat(g)
    deg = A.sum(1)
    m = int(deg.sum()) // 2
    A3 = np.linalg.matrix_power(A, 3)
    A4 = np.linalg.matrix_power(A, 4)
    triangles = int(np.trace(A3)) // 6
    c4 = (int(np.trace(A4)) - 2 * int((deg ** 2).sum()) + 2 * m) // 8
    tris = [t for t in itertools.combinations(range(n), 3)
            if A[t[0], t[1]] and A[t[0], t[2]] and A[t[1], t[2]]]
    assert len(tris) == triangles
    tailed = sum(int(deg[v]) - 2 for t in tris for v in t)
    k4 = sum(1 for t in itertools.combinations(range(n), 4)
             if all(A[a, b] for a, b in itertools.combinations(t, 2)))
    expect = {
        "vertex": n, "edge": m, "wedge": sum(comb(int(d), 2) for d in deg),
        "triangle": triangles, "cycle4": c4, "1-tailed-triangle": tailed,
        "clique4": k4,
    }
    for k in range(2, 6):
        expect[f"{k}-star"] = sum(comb(int(d), k) for d in deg)
    for name, val in expect.items():
        P = PATTERNS[name]
        assert oracle.fringe_count(g, P.n, P.edges) == val, name
        if P.n <= 5:
            assert oracle.brute_force_count(g, P.n, P.edges) == val, name
    cf = oracle.closed_forms(g)
    assert cf["edge"] == m and cf["3-star"] == expect["3-star"]
    # k-tailed triangles: explicit triples x C(deg - 2, k), vs the brute-force
    # mode (k <= 2: <= 5 pattern vertices) and the core/fringe mode
    for k in range(1, 5):
        want = sum(comb(int(deg[v]) - 2, k) for t in tris for v in t)
        assert oracle.k_tailed_triangles(g, k) == want
        P = PATTERNS[f"{k}-tailed-triangle"]
        assert oracle.fringe_count(g, P.n, P.edges) == want, k
        if P.n <= 5:
            assert oracle.brute_force_count(g, P.n, P.edges) == want, k


# ------------------------------------------------------------ exhaustive

def _all_graphs_5():
    """All graphs on 5 vertices up to isomorphism (34), incl. disconnected."""
    pairs = list(itertools.combinations(range(5), 2))
    perms = list(itertools.permutations(range(5)))
    seen, out = set(), []
    for mask in range(1 << 10):
        es = [pairs[i] for i in range(10) if mask >> i & 1]
        canon = min(tuple(sorted(tuple(sorted((p[a], p[b]))) for a, b in es)) for p in perms)
        if canon not in seen:
            seen.add(canon)
            out.append(es)
    return out


def test_exhaustive_small():
    """Sec. 3.4: "we exhaustively tested Fringe-SGC on all possible patterns
    with up to 5 vertices on all possible graphs with up to 5 vertices" --
    mode 2 (core + fringe formula) must equal mode 1 (brute force)."""
    pats = all_connected_patterns(5)
    graphs = _all_graphs_5()
    assert len(pats) == 31 and len(graphs) == 34
    for es in graphs:
        g = oracle.simple_adjacency(5, es)
        for P in pats:
            assert oracle.fringe_count(g, P.n, P.edges) == oracle.brute_force_count(g, P.n, P.edges), (P, es)


@pytest.mark.parametrize("seed", range(4))
def test_random_graphs_named_patterns(seed):
    """Brute force on small random graphs (9-11 vertices, dense enough to hold
    every pattern) for the named patterns up to 7 vertices."""
    n = 9 + seed % 3
    _, g = rand_graph(n, 0.55, 100 + seed)
    for name in ["path4", "path5", "cycle5", "clique4", "diamond", "2-tailed-triangle",
                 "3-tailed-triangle", "4-star", "k4core+1f", "diamondcore+2f",
                 "tricore+3f", "c4core+2f"]:
        P = PATTERNS[name]
        assert oracle.fringe_count(g, P.n, P.edges, P.core) == oracle.brute_force_count(g, P.n, P.edges), name


# ------------------------------------------------------------ fc pins

def _sec31_formula(nu, nv, nuv, k, l, m):
    """Sec. 3.1, last displayed formula (edge core, k tails on u, l tails on v,
    m wedge fringes)."""
    C = lambda n_, k_: comb(n_, k_) if n_ >= 0 and k_ >= 0 else 0
    tot = 0
    for i in range(k + 1):
        for j in range(l + 1):
            tot += C(nu, k - i) * C(nuv, i) * C(nv, l - j) * C(nuv - i, j) * C(nuv - i - j, m)
    return tot


def test_fc_edge_core_formulas():
    """Sec. 3.1 displayed formulas vs Listing 5 (bit 0 = u, bit 1 = v)."""
    rng = random.Random(5)
    for _ in range(400):
        nu, nv, nuv = rng.randint(0, 7), rng.randint(0, 7), rng.randint(0, 7)
        k, l, m = rng.randint(0, 4), rng.randint(0, 4), rng.randint(0, 4)
        venn = [0, nu, nv, nuv]
        anch, ks = [], []
        for a, kk in ((0b01, k), (0b10, l), (0b11, m)):
            if kk:
                anch.append(a); ks.append(kk)
        assert oracle.fc(venn, 2, anch, ks) == _sec31_formula(nu, nv, nuv, k, l, m)
        # tailed triangle: C(nu,1)C(nuv,1) + C(nuv,1)C(nuv-1,1)
        assert oracle.fc(venn, 2, [0b01, 0b11], [1, 1]) == nu * nuv + nuv * (nuv - 1)
        # 1 tail + m wedges: C(nu,1)C(nuv,m) + C(nuv,1)C(nuv-1,m)
        if m:
            assert oracle.fc(venn, 2, [0b01, 0b11], [1, m]) == nu * comb(nuv, m) + nuv * comb(max(nuv - 1, 0), m) * (nuv >= 1)
        # m wedges alone: C(c, m) ("with m wedge fringes, there will be C(c,m)")
        assert oracle.fc(venn, 2, [0b11], [m or 1]) == comb(nuv, m or 1)
    # the Sec. 3.1 identity C(n,a)C(n-a,b) = C(n-b,a)C(n,b)
    for n_ in range(8):
        for a in range(n_ + 1):
            for b in range(n_ - a + 1):
                assert comb(n_, a) * comb(n_ - a, b) == comb(n_ - b, a) * comb(n_, b)


def _fc_by_definition(venn, q, anch, ks):
    """Definition: number of tuples of pairwise disjoint sets S_t, |S_t| = k_t,
    S_t inside the union of the Venn regions covering anch_t -- on explicit
    elements, by exhaustive search (tiny sizes only)."""
    elems = []
    for idx in range(1, 1 << q):
        elems += [idx] * venn[idx]           # element = its region index
    N = len(elems)
    allowed = [[x for x in range(N) if elems[x] & a == a] for a in anch]

    def rec(t, used):
        if t == len(anch):
            return 1
        tot = 0
        for S in itertools.combinations([x for x in allowed[t] if x not in used], ks[t]):
            tot += rec(t + 1, used | set(S))
        return tot
    return rec(0, set())


def test_fc_definition_bruteforce_q3():
    """fc (Listing 5) vs the definition on explicit sets, random q<=3
    Venn diagrams, random fringe types -- catches a wrong covering-set walk
    (idx = (idx+1)|anch, Sec. 3.4), a missing restore, a wrong final entry."""
    rng = random.Random(11)
    for _ in range(300):
        q = rng.randint(1, 3)
        venn = [0] + [rng.randint(0, 3) for _ in range((1 << q) - 1)]
        ntypes = rng.randint(1, min(3, (1 << q) - 1))
        anch = rng.sample(range(1, 1 << q), ntypes)
        ks = [rng.randint(1, 3) for _ in anch]
        want = _fc_by_definition(venn, q, anch, ks)
        assert oracle.fc(list(venn), q, anch, ks) == want
        # the type order does not matter (Sec. 3.2 "we can start with any fringe type")
        perm = list(range(ntypes)); rng.shuffle(perm)
        assert oracle.fc(list(venn), q, [anch[i] for i in perm], [ks[i] for i in perm]) == want


def test_kstar_formula():
    """Sec. 3: every vertex is the centre of exactly C(d, k) k-stars."""
    for d in range(12):
        for k in range(1, 7):
            assert oracle.fc([0, d], 1, [1], [k]) == comb(d, k)


# ------------------------------------------------------------ automorphisms

def test_automorphism_counts():
    """Sec. 3.1: "a triangle has six automorphisms"; textbook values for the
    rest (|Aut(K_n)| = n!, |Aut(k-star)| = k!, |Aut(C_n)| = 2n)."""
    A = lambda name: oracle.automorphism_count(PATTERNS[name].n, PATTERNS[name].edges)
    assert A("triangle") == 6
    assert A("clique4") == 24 and A("clique5") == 120
    assert A("cycle4") == 8 and A("cycle5") == 10
    assert A("diamond") == 4 and A("path4") == 2 and A("1-tailed-triangle") == 2
    for k in range(2, 7):
        assert A(f"{k}-star") == factorial(k)
    # backtracking branch (n > 8): 8-star = 8!, and fig4 reading (DESIGN R5):
    # swap(u,w) x 2!^3 tails x 2!2!1! wedges x 2! tri-fringes
    s8 = star(8)
    assert oracle.automorphism_count(s8.n, s8.edges) == factorial(8)
    assert A("fig4") == 2 * 8 * 4 * 2


# ------------------------------------------------------------ decomposition

def test_decomposition_paper_statements():
    D = lambda name: oracle.decompose(PATTERNS[name].n, PATTERNS[name].edges)
    # Sec. 3.1 "The simplest pattern with a 2-vertex core ... is the triangle"
    d = D("triangle"); assert len(d.core) == 2 and d.types[0][1] == 1 and len(d.types[0][0]) == 2
    # Sec. 3.2: "the 4-cycle in Fig. 1 has a wedge core and the 4-clique has a triangle core"
    d = D("cycle4"); assert len(d.core) == 3
    assert sum(1 for a, b in PATTERNS["cycle4"].edges if a in d.core and b in d.core) == 2
    d = D("clique4"); assert len(d.core) == 3 and d.types == [(frozenset(d.core), 1)]
    # Sec. 3.1: tailed triangle = 2-vertex core, a wedge fringe and a tail fringe
    d = D("1-tailed-triangle"); assert len(d.core) == 2 and sorted(len(a) for a, _ in d.types) == [1, 2]
    # Sec. 3: k-stars have a single central (core) vertex
    d = D("4-star"); assert d.core == (0,) and d.types == [(frozenset({0}), 4)]
    # Sec. 1 / 3.2: Fig. 4 has a 3-vertex core and tri-fringes O and P
    d = D("fig4"); assert d.core == (0, 1, 2) and (frozenset({0, 1, 2}), 2) in d.types
    assert sum(kk for _, kk in d.types) == 13


def test_decomposition_validity_all_small():
    """Def. 3.1/3.2: for every connected pattern <= 5 vertices the heuristic
    core is connected and the non-core vertices touch only core vertices."""
    for P in all_connected_patterns(5):
        d = oracle.decompose(P.n, P.edges)
        adj = oracle.pattern_adjacency(P.n, P.edges)
        for v in range(P.n):
            if v not in d.core:
                assert adj[v] and adj[v] <= set(d.core)


def test_count_independent_of_core_choice():
    """Any valid decomposition gives the same count (Sec. 3, "the core is not
    unique"): heuristic core vs a forced larger core."""
    _, g = rand_graph(11, 0.5, 77)
    cases = [(PATTERNS["clique4"], (0, 1, 2, 3)), (PATTERNS["1-tailed-triangle"], (0, 1, 2)),
             (PATTERNS["cycle4"], (0, 1, 2, 3)), (PATTERNS["path4"], (0, 1, 2, 3)),
             (PATTERNS["diamond"], (0, 1, 2))]
    for P, core in cases:
        assert oracle.fringe_count(g, P.n, P.edges, core) == oracle.fringe_count(g, P.n, P.edges)


# ------------------------------------------------------------ CSR definition

def test_degree_ordered_csr_definition():
    rng = np.random.default_rng(3)
    n = 60
    e = rng.integers(0, n, size=(400, 2))            # duplicates + self loops
    offs, adj, order = oracle.degree_ordered_csr(n, e)
    g = oracle.simple_adjacency(n, e.tolist())
    assert sorted(order.tolist()) == list(range(n))
    degs = [len(g[order[i]]) for i in range(n)]
    assert degs == sorted(degs)
    for i in range(n - 1):
        if degs[i] == degs[i + 1]:
            assert order[i] < order[i + 1]
    rank = {int(v): i for i, v in enumerate(order)}
    for i in range(n):
        lst = adj[offs[i]:offs[i + 1]].tolist()
        assert lst == sorted(rank[w] for w in g[order[i]])
    assert offs[-1] == sum(len(s) for s in g)


# ------------------------------------------------------------ per-root sums

def test_root_raw_sum_matches_rooted_embeddings():
    """root_raw_sum(r) * prod k! = #embeddings psi with psi(root) = r
    (brute-force rooted count), and summing over r gives the total raw sum."""
    _, g = rand_graph(10, 0.5, 5)
    for name in ["1-tailed-triangle", "cycle4", "diamond", "path4", "3-star"]:
        P = PATTERNS[name]
        d = oracle.decompose(P.n, P.edges)
        scale = 1
        for _, kk in d.types:
            scale *= factorial(kk)
        total, raw = oracle.fringe_count(g, P.n, P.edges, return_raw=True)
        for root in d.core:
            acc = 0
            for r in range(len(g)):
                rr = oracle.root_raw_sum(g, P.n, P.edges, None, root, r)
                assert rr * scale == oracle.count_monomorphisms(g, P.n, P.edges, fixed=(root, r))
                acc += rr
            assert acc == raw


def test_core_matches():
    _, g = rand_graph(12, 0.45, 9)
    A = adjmat(g)
    P = PATTERNS["1-tailed-triangle"]
    assert oracle.core_matches(g, P.n, P.edges) == int(A.sum()) // 2          # edge core
    P = PATTERNS["clique4"]
    assert oracle.core_matches(g, P.n, P.edges) == int(np.trace(np.linalg.matrix_power(A, 3))) // 6


def _set_partitions(items):
    if not items:
        yield []
        return
    first, rest = items[0], items[1:]
    for p in _set_partitions(rest):
        yield [[first]] + p
        for i in range(len(p)):
            yield p[:i] + [[first] + p[i]] + p[i + 1:]


def test_partition_lattice_identity_equals_listing5():
    """The GPU evaluates fc for programs whose fringe types all have k = 1 by
    Moebius inversion on the partition lattice: #(distinct x_t in U_t) =
    sum_pi prod_B (-1)^(|B|-1) (|B|-1)! |cap_{t in B} U_t|.  Pin that identity
    against Listing 5 (oracle.fc) on random Venn diagrams, q <= 4."""
    from math import factorial
    rng = random.Random(21)
    for _ in range(250):
        q = rng.randint(1, 4)
        venn = [0] + [rng.randint(0, 4) for _ in range((1 << q) - 1)]
        s = rng.randint(1, min(5, (1 << q) - 1))
        anch = rng.sample(range(1, 1 << q), s)
        Z = {}
        for A in range(1 << q):
            Z[A] = sum(venn[e] for e in range(1, 1 << q) if e & A == A)
        tot = 0
        for part in _set_partitions(list(range(s))):
            term = 1
            for B in part:
                mask = 0
                for t in B:
                    mask |= anch[t]
                term *= (-1) ** (len(B) - 1) * factorial(len(B) - 1) * Z[mask]
            tot += term
        assert tot == oracle.fc(list(venn), q, anch, [1] * s)


# ------------------------------------------------------------ the C oracle (oracle/cfast.py)
# The C transcription of mode 2 is pinned to the pinned Python oracle on
# every small pattern, and to closed forms at sizes the Python oracle does
# not reach (RMAT graphs with hubs).

def test_c_oracle_equals_python_oracle_all_small_patterns():
    from oracle.cfast import fringe_count_c, simple_csr
    for seed in range(3):
        n = 12 + 2 * seed
        edges, g = rand_graph(n, 0.4, seed + 40)
        csr = simple_csr(n, edges)
        pats = all_connected_patterns(5) + [PATTERNS[x] for x in
                                            ("fig4", "k4core+6f", "tricore+6f", "c4core+4f", "diamondcore+5f",
                                             "4-tailed-triangle", "6-star")]
        for P in pats:
            assert fringe_count_c(csr, P.n, P.edges, P.core)[0] == oracle.fringe_count(g, P.n, P.edges, P.core), P


def test_c_oracle_root_sums_equal_python_oracle():
    from oracle.cfast import root_raw_sum_c, simple_csr
    n = 16
    edges, g = rand_graph(n, 0.35, 7)
    csr = simple_csr(n, edges)
    for name in ("tricore+3f", "1-tailed-triangle", "k4core+2f", "c4core+2f"):
        P = PATTERNS[name]
        dec = oracle.decompose(P.n, P.edges, P.core)
        for pv in dec.core:
            roots = [1, 5, 9]
            want = sum(oracle.root_raw_sum(g, P.n, P.edges, P.core, pv, r) for r in roots)
            assert root_raw_sum_c(csr, P.n, P.edges, P.core, pv, roots)[0] == want, (name, pv)


def test_c_oracle_closed_forms_on_rmat():
    """RMAT scale 11 (hubs of degree ~800): k-tailed triangles = sum over
    triangles of C(deg x - 2, k) (oracle.k_tailed_triangles, itself pinned),
    k-stars = sum C(deg, k), triangles = trace(A^3) / 6, edges = m."""
    import scipy.sparse as sp
    from inputs.graphs import rmat_edges_np
    from oracle.cfast import fringe_count_c, simple_csr
    n = 1 << 11
    e = rmat_edges_np(11, 8, seed=3)
    csr = simple_csr(n, e)
    offs, adj = csr
    g = oracle.csr_to_adjacency(offs, adj)
    deg = np.diff(offs)
    A = sp.csr_matrix((np.ones(len(adj), dtype=np.int64), adj, offs), shape=(n, n))
    tri = int((A @ A).multiply(A).sum()) // 6
    assert fringe_count_c(csr, 3, PATTERNS["triangle"].edges)[0] == tri
    assert fringe_count_c(csr, 2, PATTERNS["edge"].edges)[0] == len(adj) // 2
    for k in (2, 4):
        P = PATTERNS[f"{k}-star"]
        assert fringe_count_c(csr, P.n, P.edges)[0] == sum(comb(int(d), k) for d in deg)
    for k in (1, 3):
        P = PATTERNS[f"{k}-tailed-triangle"]
        assert fringe_count_c(csr, P.n, P.edges)[0] == oracle.k_tailed_triangles(g, k)
        # the same pattern with the triangle forced as the core (Def. 3.1: any
        # valid core gives the same count)
        assert fringe_count_c(csr, P.n, P.edges, core=(0, 1, 2))[0] == oracle.k_tailed_triangles(g, k)


def test_c_oracle_overflow_is_flagged():
    """a star with 200,000 leaves: C(200000, 9) > 2^128 must raise, C(n, 7)
    is exact"""
    from oracle.cfast import fringe_count_c, simple_csr
    L = 200000
    e = np.stack([np.zeros(L, dtype=np.int64), np.arange(1, L + 1)], axis=1)
    csr = simple_csr(L + 1, e)
    assert fringe_count_c(csr, 8, star(7).edges)[0] == comb(L, 7)
    with pytest.raises(OverflowError):
        fringe_count_c(csr, 10, star(9).edges)
