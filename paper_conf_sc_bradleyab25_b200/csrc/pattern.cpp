// pattern.cpp -- host-side pattern analysis (fsgc_compile_pattern) and the
// per-pass program builder used by fsgc_count.
//
// PAPER.md: Def. 3.1-3.3 (core, fringe vertex, anchors), Sec. 3.4 (the
// decomposition heuristic and the connectivity repair, fringe types = distinct
// anchor sets with multiplicity k), Sec. 3.1 (automorphisms / symmetry
// breaking), Sec. 3.6 (matching order: most constrained core vertex first,
// maintaining connectivity).  Not performance critical: "it only needs to be
// done once per pattern and is independent of the graph" (Sec. 3.4).
#include "internal.h"

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <set>
#include <utility>

static thread_local std::string g_last_error;

void fsgc_set_error(const char* fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
}

extern "C" const char* fsgc_last_error(void) { return g_last_error.c_str(); }
extern "C" const char* fsgc_version(void) { return "fsgc-b200 0.1 (sm_100a)"; }

static inline int popc64(uint64_t x) { return __builtin_popcountll(x); }
static inline int ctz64(uint64_t x) { return __builtin_ctzll(x); }

// vertices of `vs` reachable from `start` inside `vs`
static uint64_t reach(uint64_t vs, uint64_t start, const uint64_t* adj) {
    uint64_t seen = start, frontier = start;
    while (frontier) {
        uint64_t nxt = 0;
        for (uint64_t f = frontier; f; f &= f - 1) nxt |= adj[ctz64(f)];
        nxt &= vs & ~seen;
        seen |= nxt;
        frontier = nxt;
    }
    return seen;
}

static bool is_connected(uint64_t vs, const uint64_t* adj) {
    if (!vs) return true;
    return reach(vs, vs & (~vs + 1), adj) == vs;
}

// Sec. 3.4 heuristic: by increasing pattern degree (ties: increasing id), an
// unprocessed vertex becomes a fringe and its neighbours become core.
static uint64_t heuristic_core(int n, const uint64_t* adj) {
    std::vector<int> state(n, 0);  // 0 unprocessed, 1 fringe, 2 core
    int maxdeg = 0;
    for (int v = 0; v < n; ++v) maxdeg = std::max(maxdeg, popc64(adj[v]));
    for (int d = 0; d <= maxdeg; ++d)
        for (int v = 0; v < n; ++v)
            if (popc64(adj[v]) == d && state[v] == 0) {
                state[v] = 1;
                for (uint64_t a = adj[v]; a; a &= a - 1) state[ctz64(a)] = 2;
            }
    uint64_t core = 0;
    for (int v = 0; v < n; ++v)
        if (state[v] == 2) core |= 1ull << v;
    return core;
}

// Sec. 3.4 repair: while the core is disconnected, BFS (neighbours in
// increasing id order) from the component of the smallest core vertex until a
// vertex of another core component is reached; the path's interior joins.
static uint64_t connect_core(int n, const uint64_t* adj, uint64_t core) {
    for (;;) {
        uint64_t first = reach(core, core & (~core + 1), adj);
        if (first == core) return core;
        std::vector<int> parent(n, -2);
        std::vector<int> queue;
        for (uint64_t f = first; f; f &= f - 1) {
            int v = ctz64(f);
            parent[v] = -1;
            queue.push_back(v);
        }
        int hit = -1;
        for (size_t qi = 0; qi < queue.size() && hit < 0; ++qi) {
            int x = queue[qi];
            for (uint64_t a = adj[x]; a; a &= a - 1) {
                int y = ctz64(a);
                if (parent[y] != -2) continue;
                parent[y] = x;
                if (core >> y & 1) { hit = y; break; }
                queue.push_back(y);
            }
        }
        if (hit < 0) return 0;  // cannot happen for a connected pattern
        for (int x = parent[hit]; x >= 0 && !(first >> x & 1); x = parent[x]) core |= 1ull << x;
    }
}

static bool mul_u64(uint64_t a, uint64_t b, uint64_t* r) { return !__builtin_mul_overflow(a, b, r); }

// |Aut(P)| = prod over false-twin classes of |class|!  x  |Aut| of the
// class quotient labelled by class size (twins = equal open neighbourhoods).
static bool automorphisms(int n, const uint64_t* adj, uint64_t* out) {
    std::map<uint64_t, std::vector<int>> cls;
    for (int v = 0; v < n; ++v) cls[adj[v]].push_back(v);
    std::vector<int> size, rep;
    for (auto& kv : cls) { size.push_back((int)kv.second.size()); rep.push_back(kv.second[0]); }
    const int nc = (int)size.size();
    std::vector<int> cls_of(n);
    { int c = 0; for (auto& kv : cls) { for (int v : kv.second) cls_of[v] = c; ++c; } }
    std::vector<uint64_t> qadj(nc, 0);  // nc <= 64
    for (int c = 0; c < nc; ++c)
        for (uint64_t a = adj[rep[c]]; a; a &= a - 1) qadj[c] |= 1ull << cls_of[ctz64(a)];
    uint64_t total = 1;
    for (int c = 0; c < nc; ++c)
        for (int i = 2; i <= size[c]; ++i)
            if (!mul_u64(total, (uint64_t)i, &total)) return false;
    // labelled automorphisms of the quotient by backtracking
    std::vector<int> img(nc, -1);
    std::vector<char> used(nc, 0);
    uint64_t qaut = 0;
    bool ok = true;
    struct Rec {
        int nc; const std::vector<int>& size; const std::vector<uint64_t>& qadj;
        std::vector<int>& img; std::vector<char>& used; uint64_t& cnt; bool& ok;
        void go(int i) {
            if (!ok) return;
            if (i == nc) { if (++cnt == 0) ok = false; return; }
            for (int c = 0; c < nc; ++c) {
                if (used[c] || size[c] != size[i] || popc64(qadj[c]) != popc64(qadj[i])) continue;
                bool good = true;
                for (int j = 0; j < i && good; ++j)
                    good = (((qadj[i] >> j) & 1) == ((qadj[c] >> img[j]) & 1));
                if (good && (((qadj[i] >> i) & 1) != ((qadj[c] >> c) & 1))) good = false;
                if (!good) continue;
                used[c] = 1; img[i] = c;
                go(i + 1);
                used[c] = 0;
            }
        }
    } rec{nc, size, qadj, img, used, qaut, ok};
    rec.go(0);
    if (!ok) return false;
    return mul_u64(total, qaut, out);
}

// permutations of core positions preserving the core's edges
static std::vector<std::array<int8_t, FSGC_MAXC>> core_automorphisms(int p, const uint64_t* cadj) {
    std::vector<std::array<int8_t, FSGC_MAXC>> out;
    std::array<int8_t, FSGC_MAXC> perm{};
    for (int i = 0; i < p; ++i) perm[i] = (int8_t)i;
    do {
        bool ok = true;
        for (int i = 0; i < p && ok; ++i)
            for (int j = 0; j < p && ok; ++j)
                if (((cadj[i] >> j) & 1) != ((cadj[perm[i]] >> perm[j]) & 1)) ok = false;
        if (ok) out.push_back(perm);
    } while (std::next_permutation(perm.begin(), perm.begin() + p));
    return out;
}

static uint64_t map_mask(uint64_t m, const std::array<int8_t, FSGC_MAXC>& s) {
    uint64_t r = 0;
    for (; m; m &= m - 1) r |= 1ull << s[ctz64(m)];
    return r;
}

extern "C" int fsgc_compile_pattern(int n, const int32_t* edges, int ne, const int32_t* core,
                                    int core_size, fsgc_pattern** out) {
    if (!out) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_compile_pattern: out is NULL");
    *out = nullptr;
    if (n < 1 || n > FSGC_MAX_PATTERN_VERTICES)
        FSGC_FAIL(FSGC_ERR_INVALID, "pattern must have 1..%d vertices (got %d)", FSGC_MAX_PATTERN_VERTICES, n);
    if (ne < 0 || (ne > 0 && !edges)) FSGC_FAIL(FSGC_ERR_INVALID, "bad pattern edge list");
    if (core_size < 0 || (core_size > 0 && !core)) FSGC_FAIL(FSGC_ERR_INVALID, "bad core list");
    fsgc_pattern P;
    P.n = n;
    for (int i = 0; i < ne; ++i) {
        int a = edges[2 * i], b = edges[2 * i + 1];
        if (a < 0 || b < 0 || a >= n || b >= n) FSGC_FAIL(FSGC_ERR_INVALID, "pattern edge (%d,%d) out of range", a, b);
        if (a == b) FSGC_FAIL(FSGC_ERR_PATTERN, "pattern self loop at %d", a);
        if (P.adj[a] >> b & 1) FSGC_FAIL(FSGC_ERR_PATTERN, "duplicate pattern edge (%d,%d)", a, b);
        P.adj[a] |= 1ull << b;
        P.adj[b] |= 1ull << a;
        P.edges.push_back({a, b});
    }
    const uint64_t all = (n == 64) ? ~0ull : ((1ull << n) - 1);
    if (!is_connected(all, P.adj)) FSGC_FAIL(FSGC_ERR_PATTERN, "pattern is not connected");

    uint64_t cm = 0;
    if (n == 1) {
        cm = 1;
    } else if (core_size == 0) {
        cm = connect_core(n, P.adj, heuristic_core(n, P.adj));
    } else {
        for (int i = 0; i < core_size; ++i) {
            if (core[i] < 0 || core[i] >= n) FSGC_FAIL(FSGC_ERR_INVALID, "core vertex %d out of range", core[i]);
            cm |= 1ull << core[i];
        }
        if (!is_connected(cm, P.adj)) FSGC_FAIL(FSGC_ERR_PATTERN, "given core is not connected");
        for (int v = 0; v < n; ++v)
            if (!(cm >> v & 1) && (P.adj[v] & ~cm))
                FSGC_FAIL(FSGC_ERR_PATTERN, "non-core vertex %d is adjacent to a non-core vertex (Def. 3.1)", v);
    }
    const int p = popc64(cm);
    if (p < 1 || p > FSGC_MAX_CORE) FSGC_FAIL(FSGC_ERR_PATTERN, "core has %d vertices (limit %d)", p, FSGC_MAX_CORE);
    P.core_mask = cm;

    // fringe types: distinct anchor sets (Def. 3.3), grouped, ascending mask
    std::map<uint64_t, int> types;
    for (int v = 0; v < n; ++v)
        if (!(cm >> v & 1)) types[P.adj[v]] += 1;
    for (auto& kv : types) {
        P.type_anchor.push_back(kv.first);
        P.type_k.push_back(kv.second);
    }

    // matching order (Sec. 3.6): most constrained first, keep connectivity
    uint64_t placed = 0;
    for (int it = 0; it < p; ++it) {
        int best = -1;
        long bestkey = -1;
        for (uint64_t c = cm & ~placed; c; c &= c - 1) {
            int v = ctz64(c);
            int back = popc64(P.adj[v] & placed);
            if (it > 0 && back == 0) continue;
            long key = (long)back * 4096 + popc64(P.adj[v]) * 64 + (63 - v);
            if (key > bestkey) { bestkey = key; best = v; }
        }
        if (best < 0) FSGC_FAIL(FSGC_ERR_INTERNAL, "matching order failed");
        P.order.push_back(best);
        placed |= 1ull << best;
    }

    if (!automorphisms(n, P.adj, &P.aut))
        FSGC_FAIL(FSGC_ERR_PATTERN, "|Aut(P)| exceeds 2^64");
    for (int k : P.type_k)
        for (int i = 2; i <= k; ++i)
            if (!mul_u64(P.fringe_fact, (uint64_t)i, &P.fringe_fact))
                FSGC_FAIL(FSGC_ERR_PATTERN, "prod k! exceeds 2^64");

    // core automorphisms, unlabeled and fringe-labelled
    uint64_t cadj[FSGC_MAXC] = {};
    int posof[FSGC_MAX_PATTERN_VERTICES];
    for (int i = 0; i < p; ++i) posof[P.order[i]] = i;
    for (int i = 0; i < p; ++i)
        for (int j = 0; j < p; ++j)
            if (P.adj[P.order[i]] >> P.order[j] & 1) cadj[i] |= 1ull << j;
    std::vector<std::pair<uint64_t, int>> tpos;
    for (size_t t = 0; t < P.type_anchor.size(); ++t) {
        uint64_t m = 0;
        for (uint64_t a = P.type_anchor[t]; a; a &= a - 1) m |= 1ull << posof[ctz64(a)];
        tpos.push_back({m, P.type_k[t]});
    }
    std::sort(tpos.begin(), tpos.end());
    auto autos = core_automorphisms(p, cadj);
    P.aut_core = autos.size();
    P.aut_core_labeled = 0;
    for (auto& s : autos) {
        std::vector<std::pair<uint64_t, int>> img;
        for (auto& t : tpos) img.push_back({map_mask(t.first, s), t.second});
        std::sort(img.begin(), img.end());
        if (img == tpos) P.aut_core_labeled++;
    }
    static std::atomic<uint64_t> next_uid{1};
    P.uid = next_uid.fetch_add(1);
    *out = new fsgc_pattern(P);
    return FSGC_OK;
}

extern "C" int fsgc_pattern_get_info(const fsgc_pattern* p, fsgc_pattern_info* o) {
    if (!p || !o) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_pattern_get_info: null argument");
    std::memset(o, 0, sizeof *o);
    o->num_vertices = p->n;
    o->num_edges = (int)p->edges.size();
    o->core_size = (int)p->order.size();
    for (size_t i = 0; i < p->order.size(); ++i) o->core_order[i] = p->order[i];
    o->num_types = (int)p->type_anchor.size();
    for (size_t t = 0; t < p->type_anchor.size(); ++t) {
        o->type_anchor[t] = p->type_anchor[t];
        o->type_count[t] = p->type_k[t];
    }
    o->core_mask = p->core_mask;
    o->aut = p->aut;
    o->aut_core = p->aut_core;
    o->aut_core_labeled = p->aut_core_labeled;
    o->fringe_factorial = p->fringe_fact;
    return FSGC_OK;
}

extern "C" void fsgc_free_pattern(fsgc_pattern* p) { delete p; }

// --------------------------------------------------------------- passes

static void position_adjacency(const fsgc_pattern* P, uint64_t* cadj) {
    const int p = (int)P->order.size();
    for (int i = 0; i < p; ++i) {
        cadj[i] = 0;
        for (int j = 0; j < p; ++j)
            if (P->adj[P->order[i]] >> P->order[j] & 1) cadj[i] |= 1ull << j;
    }
}

// Map `other`'s core onto `ref`'s core positions (pos_of[pattern vertex] =
// position, -1 off-core).  Returns 1 if the cores are isomorphic.
int fsgc_core_isomorphism(const fsgc_pattern* ref, const fsgc_pattern* other, int* pos_of) {
    const int p = (int)ref->order.size();
    if ((int)other->order.size() != p) return 0;
    uint64_t ra[FSGC_MAXC], oa[FSGC_MAXC];
    position_adjacency(ref, ra);
    position_adjacency(other, oa);
    std::array<int8_t, FSGC_MAXC> perm{};
    for (int i = 0; i < p; ++i) perm[i] = (int8_t)i;
    do {  // other's position i -> ref position perm[i]
        bool ok = true;
        for (int i = 0; i < p && ok; ++i)
            for (int j = 0; j < p && ok; ++j)
                if (((oa[i] >> j) & 1) != ((ra[perm[i]] >> perm[j]) & 1)) ok = false;
        if (ok) {
            for (int v = 0; v < FSGC_MAX_PATTERN_VERTICES; ++v) pos_of[v] = -1;
            for (int i = 0; i < p; ++i) pos_of[other->order[i]] = perm[i];
            return 1;
        }
    } while (std::next_permutation(perm.begin(), perm.begin() + p));
    return 0;
}

int fsgc_build_pass(const fsgc_pattern* const* pats, const std::vector<int>& members,
                    int nosym, PassPlan* plan) {
    const fsgc_pattern* ref = pats[members[0]];
    const int p = (int)ref->order.size();
    CoreProg& cp = plan->prog;
    std::memset(&cp, 0, sizeof cp);
    plan->members = members;
    plan->divisor.clear();
    cp.p = p;
    cp.npats = (int)members.size();
    if (cp.npats > FSGC_MAXPATS) FSGC_FAIL(FSGC_ERR_INVALID, "too many patterns in one pass");

    uint64_t cadj[FSGC_MAXC];
    position_adjacency(ref, cadj);
    for (int i = 1; i < p; ++i) {
        cp.back[i] = (uint8_t)(cadj[i] & ((1ull << i) - 1));
        if (!cp.back[i]) FSGC_FAIL(FSGC_ERR_INTERNAL, "matching order not connected");
    }
    auto autos = core_automorphisms(p, cadj);

    // symmetry breaking restrictions from the stabiliser chain of Aut(C):
    // phi(i) < phi(j) for every j != i in the orbit of i under the pointwise
    // stabiliser of positions 0..i-1 (Sec. 3.1 "enforcing that the unique
    // vertex ID of A must be smaller than B's")
    if (!nosym) {
        std::vector<std::array<int8_t, FSGC_MAXC>> G = autos;
        for (int i = 0; i < p; ++i) {
            uint64_t orbit = 0;
            for (auto& s : G) orbit |= 1ull << s[i];
            for (uint64_t o = orbit & ~(1ull << i); o; o &= o - 1) cp.gt[ctz64(o)] |= (uint8_t)(1u << i);
            std::vector<std::array<int8_t, FSGC_MAXC>> H;
            for (auto& s : G)
                if (s[i] == i) H.push_back(s);
            G.swap(H);
        }
    }

    // fringe programs
    struct Prog { int pat; std::vector<std::pair<uint64_t, int>> types; };
    std::vector<Prog> progs;
    uint64_t anchor_union = 0;
    for (size_t mi = 0; mi < members.size(); ++mi) {
        const fsgc_pattern* P = pats[members[mi]];
        int pos_of[FSGC_MAX_PATTERN_VERTICES];
        if (!fsgc_core_isomorphism(ref, P, pos_of)) FSGC_FAIL(FSGC_ERR_INTERNAL, "cores not isomorphic");
        plan->root_pattern_vertex[mi] = -1;
        for (int v = 0; v < P->n; ++v)
            if (pos_of[v] == 0) plan->root_pattern_vertex[mi] = v;
        std::vector<std::pair<uint64_t, int>> base;
        for (size_t t = 0; t < P->type_anchor.size(); ++t) {
            uint64_t m = 0;
            for (uint64_t a = P->type_anchor[t]; a; a &= a - 1) m |= 1ull << pos_of[ctz64(a)];
            base.push_back({m, P->type_k[t]});
        }
        std::sort(base.begin(), base.end());
        std::set<std::vector<std::pair<uint64_t, int>>> distinct;
        if (nosym) {
            distinct.insert(base);
        } else {
            for (auto& s : autos) {
                std::vector<std::pair<uint64_t, int>> img;
                for (auto& t : base) img.push_back({map_mask(t.first, s), t.second});
                std::sort(img.begin(), img.end());
                distinct.insert(img);
            }
        }
        uint64_t aut_lab = nosym ? 1 : autos.size() / distinct.size();
        uint64_t denom;
        if (!mul_u64(aut_lab, P->fringe_fact, &denom) || P->aut % denom)
            FSGC_FAIL(FSGC_ERR_INTERNAL, "automorphism bookkeeping inconsistent");
        plan->divisor.push_back(P->aut / denom);
        for (auto& d : distinct) {
            progs.push_back({(int)mi, d});
            for (auto& t : d) anchor_union |= t.first;
        }
    }
    if ((int)progs.size() > FSGC_MAXPROG) FSGC_FAIL(FSGC_ERR_PATTERN, "too many fringe programs in one pass");
    cp.nprog = (int)progs.size();
    cp.q = popc64(anchor_union);
    if (cp.q > FSGC_MAXQ) FSGC_FAIL(FSGC_ERR_PATTERN, "%d anchor vertices (limit %d)", cp.q, FSGC_MAXQ);
    int bit_of[FSGC_MAXC];
    {
        int b = 0;
        for (int i = 0; i < p; ++i)
            if (anchor_union >> i & 1) { cp.anchor_pos[b] = (int8_t)i; bit_of[i] = b++; }
    }
    for (int i = 0; i < p; ++i) cp.mindeg[i] = 1 << 30;
    for (size_t k = 0; k < progs.size(); ++k) {
        FringeProg& fp = cp.prog[k];
        fp.pat = (uint8_t)progs[k].pat;
        if (progs[k].types.size() > FSGC_MAXT) FSGC_FAIL(FSGC_ERR_PATTERN, "too many fringe types");
        fp.s = (uint8_t)progs[k].types.size();
        int depth = 0, ksum = 0;
        int att[FSGC_MAXC] = {};
        // fc is independent of the fringe-type order (Sec. 3.2 "we can start
        // with any fringe type"); most constrained (largest anchor set) first
        // makes infeasible programs fail at the first, smallest Venn entries
        std::vector<std::pair<uint64_t, int>> ts = progs[k].types;
        std::stable_sort(ts.begin(), ts.end(), [](const std::pair<uint64_t, int>& a, const std::pair<uint64_t, int>& b) {
            return popc64(a.first) > popc64(b.first);
        });
        for (size_t t = 0; t < ts.size(); ++t) {
            uint64_t m = ts[t].first;
            int kk = ts[t].second;
            if (kk > 255) FSGC_FAIL(FSGC_ERR_PATTERN, "more than 255 fringes of one type");
            uint8_t vb = 0;
            for (uint64_t a = m; a; a &= a - 1) { vb |= (uint8_t)(1u << bit_of[ctz64(a)]); att[ctz64(a)] += kk; }
            fp.anch[t] = vb;
            fp.k[t] = (uint8_t)kk;
            depth += 1 << (cp.q - popc64(vb));
            ksum += kk;
            if (p == 2) {
                if (m == 1) cp.ek[k] = (uint8_t)kk;
                else if (m == 2) cp.el[k] = (uint8_t)kk;
                else cp.em[k] = (uint8_t)kk;
            }
        }
        if (depth > FSGC_FC_STACK) FSGC_FAIL(FSGC_ERR_PATTERN, "fringe program too deep (%d)", depth);
        if (ksum > 255) FSGC_FAIL(FSGC_ERR_PATTERN, "more than 255 fringes");
        fp.depth = (uint8_t)depth;
        fp.ksum = (uint8_t)ksum;
        for (int i = 0; i < p; ++i) cp.mindeg[i] = std::min(cp.mindeg[i], att[i]);
    }
    for (int i = 0; i < p; ++i) cp.mindeg[i] += popc64(cadj[i]);
    // partition-lattice term tables for programs with all k = 1 and <= 7 types
    plan->terms.assign(cp.nprog, {});
    for (int k = 0; k < cp.nprog; ++k) {
        const FringeProg& fp = cp.prog[k];
        bool ones = fp.s >= 1 && fp.s <= 7;
        for (int t = 0; t < fp.s && ones; ++t) ones = fp.k[t] == 1;
        if (!ones) continue;
        const int sN = fp.s;
        std::map<std::vector<uint8_t>, int64_t> acc;
        int rgs[7] = {0};   // restricted growth string
        for (;;) {
            int nb = 0;
            for (int i = 0; i < sN; ++i) nb = std::max(nb, rgs[i] + 1);
            std::vector<uint8_t> masks(nb, 0);
            std::vector<int> sz(nb, 0);
            for (int i = 0; i < sN; ++i) { masks[rgs[i]] |= fp.anch[i]; sz[rgs[i]]++; }
            int64_t coef = 1;
            for (int b = 0; b < nb; ++b) {
                int64_t f = 1;
                for (int j = 2; j < sz[b]; ++j) f *= j;
                coef *= ((sz[b] - 1) & 1) ? -f : f;
            }
            std::sort(masks.begin(), masks.end());
            acc[masks] += coef;
            // next restricted growth string
            int i = sN - 1;
            for (; i > 0; --i) {
                int mx = 0;
                for (int j = 0; j < i; ++j) mx = std::max(mx, rgs[j]);
                if (rgs[i] <= mx) { ++rgs[i]; break; }
                rgs[i] = 0;
            }
            if (i == 0) break;
            for (int j = i + 1; j < sN; ++j) rgs[j] = 0;
        }
        for (auto& kv : acc) {
            if (kv.second == 0) continue;
            PartTerm tm{};
            tm.coef = (int32_t)kv.second;
            tm.nb = (uint8_t)kv.first.size();
            for (size_t b = 0; b < kv.first.size(); ++b) tm.mask[b] = kv.first[b];
            plan->terms[k].push_back(tm);
        }
    }
    if (p == 1) cp.root_mode = ROOT_VERTEX;
    else if (cp.gt[1] & 1) cp.root_mode = ROOT_ORIENTED;
    else cp.root_mode = ROOT_DIRECTED;
    return FSGC_OK;
}
