"""Named query patterns (small undirected graphs) used by tests and bench.

A pattern is just vertices 0..n-1 and an edge list, plus an optional ``core``
(a set of pattern vertices) for the configs that name the core explicitly
("4-clique and diamond cores ...", BASELINE.json configs[2], configs[4]).
With ``core=None`` the code under test derives the core itself with the
PAPER.md Sec. 3.4 heuristic.  No counting arithmetic lives here.
"""
from dataclasses import dataclass, field
from typing import List, Optional, Tuple


@dataclass(frozen=True)
class Pattern:
    name: str
    n: int
    edges: Tuple[Tuple[int, int], ...]
    core: Optional[Tuple[int, ...]] = None
    note: str = field(default="", compare=False)


def _p(name, n, edges, core=None, note=""):
    return Pattern(name, n, tuple(tuple(e) for e in edges),
                   None if core is None else tuple(sorted(core)), note)


def star(k):
    """k-star: centre 0 with k spokes (Sec. 3, first paragraph)."""
    return _p(f"{k}-star", k + 1, [(0, i) for i in range(1, k + 1)])


def k_tailed_triangle(k):
    """Triangle 0-1-2 with k tails on vertex 0 (Fig. 3; reading R4 in
    DESIGN.md: all k tails share one triangle vertex, the Sec. 3.1 case
    "k tails attached to one core vertex and m wedge fringes" with m = 1)."""
    e = [(0, 1), (0, 2), (1, 2)] + [(0, 3 + i) for i in range(k)]
    return _p("triangle" if k == 0 else f"{k}-tailed-triangle", 3 + k, e)


def path(n):
    return _p(f"path{n}", n, [(i, i + 1) for i in range(n - 1)])


def cycle(n):
    return _p(f"cycle{n}", n, [(i, (i + 1) % n) for i in range(n)])


def clique(n):
    return _p(f"clique{n}", n, [(i, j) for i in range(n) for j in range(i + 1, n)])


DIAMOND_EDGES = [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3)]  # 0,1 degree 3; 2,3 degree 2


def fig4():
    """PAPER.md Fig. 4: 16 vertices, 25 edges, 3-vertex (triangle) core, tri-
    fringes O and P.  The figure is not in the extracted text; reading R5 in
    DESIGN.md: triangle u=0, v=1, w=2 with 2 tails on each core vertex, wedge
    fringes 2 on {u,v}, 2 on {v,w}, 1 on {u,w}, and 2 tri-fringes
    (3 + 6 + 2*5 + 3*2 = 25 edges, 3 + 6 + 5 + 2 = 16 vertices)."""
    e = [(0, 1), (1, 2), (0, 2)]
    nxt = 3

    def add(anchors, count):
        nonlocal nxt
        for _ in range(count):
            for a in anchors:
                e.append((a, nxt))
            nxt += 1
    add((0,), 2); add((1,), 2); add((2,), 2)
    add((0, 1), 2); add((1, 2), 2); add((0, 2), 1)
    add((0, 1, 2), 2)
    assert nxt == 16 and len(e) == 25
    return _p("fig4", 16, e)


# fringe sequence for the forced 4-vertex cores (configs[2]): single- and
# two-vertex attachment sets, added in this order
_MIXED_FRINGES = [(0,), (1, 2), (3,), (0, 3), (1,), (2, 3)]


def core_with_fringes(core_name, core_edges, core_n, nfringes, fringe_seq=_MIXED_FRINGES):
    e = list(core_edges)
    nxt = core_n
    for anchors in fringe_seq[:nfringes]:
        for a in anchors:
            e.append((a, nxt))
        nxt += 1
    return _p(f"{core_name}+{nfringes}f", nxt, e, core=range(core_n))


def k4_core(nf):
    return core_with_fringes("k4core", clique(4).edges, 4, nf)


def diamond_core(nf):
    return core_with_fringes("diamondcore", DIAMOND_EDGES, 4, nf)


def triangle_core(nf):
    """triangle core (forced) + fringes: tails and wedges on the triangle."""
    seq = [(0,), (1,), (2,), (0, 1), (1, 2), (0, 1, 2)]
    return core_with_fringes("tricore", [(0, 1), (1, 2), (0, 2)], 3, nf, seq)


def ktt_tricore(k):
    """the k-tailed triangle with its triangle FORCED as the core (DESIGN.md
    R7, R13): k tails on vertex 0, one fringe type, anchor set {0}."""
    e = [(0, 1), (0, 2), (1, 2)] + [(0, 3 + i) for i in range(k)]
    return _p(f"{k}-tailed-triangle/tricore", 3 + k, e, core=(0, 1, 2))


def c4_core(nf):
    """4-cycle core 0-1-2-3 (forced) + fringes (configs[4])."""
    seq = [(0,), (1,), (2,), (3,), (0, 2), (1, 3)]
    return core_with_fringes("c4core", cycle(4).edges, 4, nf, seq)


def _build():
    P = {}

    def put(p):
        P[p.name] = p
    put(_p("vertex", 1, []))
    put(_p("edge", 2, [(0, 1)]))
    for k in range(2, 7):
        put(star(k))
    put(_p("wedge", 3, [(0, 1), (0, 2)]))
    for k in range(0, 5):
        put(k_tailed_triangle(k))
    put(path(4)); put(path(5))
    put(cycle(4)); put(cycle(5))
    put(clique(4)); put(clique(5))
    put(_p("diamond", 4, DIAMOND_EDGES))
    put(fig4())
    for nf in range(1, 7):
        put(k4_core(nf)); put(diamond_core(nf)); put(triangle_core(nf)); put(c4_core(nf))
    for k in range(2, 5):
        put(ktt_tricore(k))
    put(_p("triangle/tricore", 3, [(0, 1), (0, 2), (1, 2)], core=(0, 1, 2)))
    put(_p("diamond/tricore", 4, DIAMOND_EDGES, core=(0, 1, 2)))
    return P


PATTERNS = _build()


def get_pattern(name) -> Pattern:
    return PATTERNS[name]


# the bench / config pattern sets (BASELINE.json configs)
CONFIG_PATTERNS = {
    "pl2k": ["1-tailed-triangle"],
    "internet": [f"{k}-tailed-triangle" for k in range(1, 5)],
    "rmat22": ["triangle", "diamond"] + [f"{k}-tailed-triangle" for k in range(1, 5)],
    "rmat16": [f"k4core+{f}f" for f in range(1, 7)] + ["diamondcore+1f"],
    "pl10m": ["fig4"],
    # configs[4]: triangle cores with fringes on RMAT-26, the core FORCED to
    # the triangle (R13): every fringe set whose Venn diagram needs
    # no triple intersection (tails, wedges on two core vertices) -- one
    # listing pass over the 4.9e10 triangles for all of them
    "rmat26": ["triangle/tricore", "tricore+1f", "tricore+2f", "2-tailed-triangle/tricore",
               "3-tailed-triangle/tricore", "4-tailed-triangle/tricore", "diamond/tricore"],
    # the same patterns decomposed by the Sec. 3.4 heuristic (edge core)
    "rmat26-edge": ["triangle"] + [f"{k}-tailed-triangle" for k in range(1, 5)],
    # the configs[4] triangle-core set on the configs[2] graph (the headline
    # pass at a second scale)
    "rmat22-tri": ["triangle/tricore", "tricore+1f", "tricore+2f", "2-tailed-triangle/tricore",
                   "3-tailed-triangle/tricore", "4-tailed-triangle/tricore", "diamond/tricore"],
    "rmat26-forced-cores": [f"tricore+{f}f" for f in range(1, 7)] + [f"c4core+{f}f" for f in range(1, 7)],
}


def all_connected_patterns(max_n) -> List[Pattern]:
    """Every connected graph on 1..max_n vertices up to isomorphism (brute
    force canonical form; max_n <= 5 gives 1+1+2+6+21 = 31 patterns).  Used for
    the PAPER.md Sec. 3.4 exhaustive check "all possible patterns with up to 5
    vertices on all possible graphs with up to 5 vertices"."""
    from itertools import combinations, permutations
    out = []
    for n in range(1, max_n + 1):
        pairs = list(combinations(range(n), 2))
        seen = set()
        perms = list(permutations(range(n)))
        for mask in range(1 << len(pairs)):
            es = [pairs[i] for i in range(len(pairs)) if mask >> i & 1]
            # connectivity
            adj = {v: set() for v in range(n)}
            for a, b in es:
                adj[a].add(b); adj[b].add(a)
            stack, vis = [0], {0}
            while stack:
                x = stack.pop()
                for y in adj[x]:
                    if y not in vis:
                        vis.add(y); stack.append(y)
            if len(vis) != n:
                continue
            canon = min(tuple(sorted(tuple(sorted((p[a], p[b]))) for a, b in es)) for p in perms)
            if canon in seen:
                continue
            seen.add(canon)
            out.append(_p(f"conn{n}_{len(seen)}", n, list(canon)))
    return out
