// count.cu -- fsgc_count: the data-parallel hot path of Fringe-SGC on sm_100a.
//
// PAPER.md Sec. 3.3-3.6 and Listing 5 (Fig. 5), Listing 7:
//   * core matching: depth-first search for the core from each root item
//     (root edge (c0,c1) or root vertex), one warp per root, the warp-ballot
//     scheme of Listing 7 ("the 32 warp threads concurrently process 32
//     vertices ... all lanes process the first such vertex together"),
//     symmetry breaking on degree-ordered ids (Sec. 3.1), degree filtering;
//   * Venn diagram: for each anchor vertex, the warp scans its sorted
//     adjacency list and binary-searches the anchors later in the order
//     (Sec. 3.6 "we search the adjacency lists of the anchor vertices that
//     appear later in the stack ... with binary search"), histograms the
//     membership bitsets, then corrects the counts for the earlier anchors and
//     excludes the matched core vertices;
//   * fringe counting: up to 32 Venn diagrams are buffered per warp, then the
//     lanes evaluate the iterative form of Listing 5 on (diagram, program)
//     pairs ("each lane runs the iterative fc function");
//   * exact 128-bit accumulation, warp-shuffle reduction, one 128-bit atomic
//     per warp and pattern.
// Work distribution: persistent CTAs, a global atomic chunk queue, heavy
// (high-degree, late in degree order) roots handed out first; shards deal
// chunks round-robin across GPUs.
#include <algorithm>
#include <cstring>
#include <map>
#include <memory>
#include <set>
#include <mutex>
#include <tuple>
#include <string>
#include <cstdlib>
#include <cstdio>
#include <cmath>
#include <functional>
#include "count_dev.cuh"

namespace {

// SM count of the current device (cached per device)
int sm_count() {
    static std::mutex mu;
    static std::map<int, int> cache;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    auto it = cache.find(dev);
    if (it != cache.end()) return it->second;
    int n = 0;
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
    cache[dev] = n;
    return n;
}

// tuning knobs (environment, read once): experiments only, defaults are the
// tuned values
int tune(const char* name, int dflt) {
    static std::mutex mu;
    static std::map<std::string, int> cache;
    std::lock_guard<std::mutex> lock(mu);
    auto it = cache.find(name);
    if (it != cache.end()) return it->second;
    const char* v = getenv(name);
    int r = v ? atoi(v) : dflt;
    cache[name] = r;
    return r;
}

// resident blocks per SM of a kernel on the current device (cached per
// device / function / block / smem); raises the kernel's dynamic shared
// memory opt-in on that device first (cudaFuncSetAttribute is per device).
// 0 when the opt-in fails (the launch would fail: the caller reports it).
int occupancy(const void* fn, int threads, size_t smem) {
    static std::mutex mu;
    static std::map<std::tuple<int, const void*, int, size_t>, int> cache;
    static std::map<std::pair<int, const void*>, size_t> optin;
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lock(mu);
    auto key = std::make_tuple(dev, fn, threads, smem);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    // the opt-in limit only grows (a plan with less shared memory must not
    // lower it below what an earlier plan of the same kernel launches with)
    size_t& lim = optin[std::make_pair(dev, fn)];
    if (smem > lim) {   // (static + dynamic above 48 KB needs the opt-in)
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess) {
            cudaGetLastError();
            return 0;
        }
        lim = smem;
    }
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, threads, smem) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    n = std::max(n, 1);
    cache[key] = n;
    return n;
}

// kernel instantiations per accumulator class (count_np.cu, one object per NP)
}  // namespace
#define FSGC_NP_DECL(NPV) const void* fsgc_np_kernel_##NPV(int which); int fsgc_np_init_##NPV();
FSGC_NP_DECL(1) FSGC_NP_DECL(2) FSGC_NP_DECL(4) FSGC_NP_DECL(8) FSGC_NP_DECL(16)
#undef FSGC_NP_DECL
namespace {

// smallest NP in {1,2,4,8,16} holding npats
int np_class(int npats) { return npats <= 1 ? 1 : npats <= 2 ? 2 : npats <= 4 ? 4 : npats <= 8 ? 8 : 16; }

// which: 0 vertex, 1 edge, 2 general core, 3 triangle core (warp tables),
// 4 triangle core (block tables)
const void* np_kernel(int which, int np) {
    switch (np) {
        case 1: return fsgc_np_kernel_1(which);
        case 2: return fsgc_np_kernel_2(which);
        case 4: return fsgc_np_kernel_4(which);
        case 8: return fsgc_np_kernel_8(which);
        default: return fsgc_np_kernel_16(which);
    }
}
const void* kernel_for(int kind, int np) { return np_kernel(kind, np); }
// triangle-core listing kernel: warp or block tables, every fc path or Z-only
const void* tri_kernel(bool zonly, bool block, int np) { return np_kernel((zonly ? 5 : 3) + (block ? 1 : 0), np); }

// hash bits of a block table holding out-degree `maxout` at load <= 1/2
int table_hbits(int64_t maxout) {
    int hb = 5;
    while ((1ll << hb) < 2 * maxout) ++hb;
    return hb;
}

}  // namespace

static int64_t roots_for(const fsgc_graph* g, int root_mode) {
    switch (root_mode) {
        case ROOT_VERTEX: return g->n;
        case ROOT_ORIENTED: return g->m;
        default: return 2 * g->m;
    }
}

extern "C" int fsgc_finalize(fsgc_u128 raw, uint64_t divisor, int32_t overflow, fsgc_u128* count,
                             int32_t* count_overflow) {
    if (!count || !count_overflow || divisor == 0) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_finalize: bad argument");
    u128 r = u128_make(raw.lo, raw.hi);
    if (!overflow && (r % divisor) != 0)
        FSGC_FAIL(FSGC_ERR_INTERNAL, "raw sum not divisible by the automorphism divisor");
    u128 c = r / divisor;
    count->lo = u128_lo(c);
    count->hi = u128_hi(c);
    *count_overflow = overflow ? 1 : 0;
    return FSGC_OK;
}

// group patterns with isomorphic cores (one pass each)
static std::vector<std::vector<int>> group_patterns(const fsgc_pattern* const* pats, int npats) {
    std::vector<std::vector<int>> groups;
    int pos_of[FSGC_MAX_PATTERN_VERTICES];
    for (int i = 0; i < npats; ++i) {
        bool placed = false;
        for (auto& gr : groups)
            if (fsgc_core_isomorphism(pats[gr[0]], pats[i], pos_of)) { gr.push_back(i); placed = true; break; }
        if (!placed) groups.push_back({i});
    }
    return groups;
}

extern "C" int fsgc_num_roots(const fsgc_graph* g, const fsgc_pattern* p, int nosym, int64_t* out) {
    if (!g || !p || !out) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_num_roots: null argument");
    PassPlan plan;
    std::vector<int> mem{0};
    const fsgc_pattern* arr[1] = {p};
    int rc = fsgc_build_pass(arr, mem, nosym, &plan);
    if (rc) return rc;
    *out = roots_for(g, plan.prog.root_mode);
    return FSGC_OK;
}

// pattern-only pass plans (groups, fringe programs), cached by pattern uid
static int pass_plans(const fsgc_pattern* const* pats, int npats, int nosym, std::vector<PassPlan>* out) {
    std::vector<uint64_t> key;
    for (int i = 0; i < npats; ++i) key.push_back(pats[i]->uid);
    key.push_back(nosym ? 1 : 0);
    static std::mutex mu;
    static std::map<std::vector<uint64_t>, std::vector<PassPlan>> cache;
    std::lock_guard<std::mutex> lock(mu);
    auto it = cache.find(key);
    if (it != cache.end()) { *out = it->second; return FSGC_OK; }
    std::vector<std::vector<int>> passes;
    for (auto& grp : group_patterns(pats, npats)) {
        std::vector<int> cur;
        for (int idx : grp) {
            std::vector<int> trial = cur;
            trial.push_back(idx);
            PassPlan probe;
            if (!cur.empty() && fsgc_build_pass(pats, trial, nosym, &probe) != FSGC_OK) {
                passes.push_back(cur);
                cur = {idx};
            } else {
                cur = trial;
            }
        }
        if (!cur.empty()) passes.push_back(cur);
    }
    std::vector<PassPlan> plans;
    for (auto& members : passes) {
        PassPlan plan;
        int rc = fsgc_build_pass(pats, members, nosym, &plan);
        if (rc) return rc;
        plans.push_back(plan);
    }
    if (cache.size() > 1024) cache.clear();
    cache[key] = plans;
    *out = plans;
    return FSGC_OK;
}

// binomial table, once per device (host-synchronous; done at plan creation so
// that enqueue stays capturable)
static int ensure_binom_table(int dev) {
    static std::mutex mu;
    static std::set<int> ready;
    std::lock_guard<std::mutex> lock(mu);
    if (ready.count(dev)) return FSGC_OK;
    int rc = dev_consts_init();   // this TU's tables (support kernels), then every NP object's
    if (!rc) rc = fsgc_np_init_1();
    if (!rc) rc = fsgc_np_init_2();
    if (!rc) rc = fsgc_np_init_4();
    if (!rc) rc = fsgc_np_init_8();
    if (!rc) rc = fsgc_np_init_16();
    if (rc) FSGC_FAIL(rc, "constant table initialisation failed: %s", cudaGetErrorString(cudaGetLastError()));
    FSGC_CUDA(cudaDeviceSynchronize());
    ready.insert(dev);
    return FSGC_OK;
}

namespace {
constexpr size_t kRawPassBytes = sizeof(AccDev) * FSGC_MAXPATS + 16;   // acc[16] | matches | pad
constexpr size_t kHdrBytes = 1024;                                      // acc | counters

struct PassExec {
    PassPlan plan;
    int kind = 0;              // 0 vertex, 1 edge (support + fc), 2 general core
    int npc = 1;               // accumulator width class
    bool zonly = false;        // triangle cores: Z-term-only listing kernels (no leaf can leave the 128-bit tier)
    int nwb2 = 8;              // triangle cores: warps per block of the block-table kernel
    int64_t grid = 1;
    size_t smem = 0;
    WorkDesc W{};
    bool uses_sup = false;     // reads the plan's per-edge support array
    size_t ws_off = 0, parts_off = 0, bytes = 0;
    int term_base = 0;         // index of this pass's programs in the term offset/count arrays
    bool whole = true;
    EdgeTerms et{};            // edge cores: the Sec. 3.1 term table (et.n == 0: checked path)
    size_t smem_fc = 0;        // dynamic shared memory of edge_fc_kernel
    VennDev vd{};              // triangle / general cores: the Venn term table (vd.n == 0: off)
    size_t smem_vd = 0;        // its per-thread binomial rows (dynamic shared memory)
    int64_t grid2 = 0;         // triangle cores: the block-table launch ...
    size_t smem2 = 0;          // ... its shared memory
    int hbits2 = 5;            // ... and table hash bits
};

// the term table of an edge-core pass (see EdgeTerms); et.n = 0 when a
// coefficient, the row length or the number of terms exceeds the table limits
static void build_edge_terms(const CoreProg& cp, EdgeTerms* et) {
    std::memset(et, 0, sizeof *et);
    std::map<std::tuple<int, int, int, int>, u128> acc;   // (pat, a, b, c) -> coef
    int ka = 0, kb = 0, kc = 0, kmax = 0;
    auto fact = [](int x) { u128 f = 1; for (int i = 2; i <= x; ++i) f *= (u128)i; return f; };
    for (int pi = 0; pi < cp.nprog; ++pi) {
        const int k = cp.ek[pi], l = cp.el[pi], m = cp.em[pi];
        if (k + l + m > 30) return;                       // (i+j+m)! must fit 128 bits
        kmax = std::max(kmax, (int)cp.prog[pi].ksum);
        for (int i = 0; i <= k; ++i)
            for (int j = 0; j <= l; ++j) {
                const u128 coef = fact(i + j + m) / (fact(i) * fact(j) * fact(m));
                acc[std::make_tuple((int)cp.prog[pi].pat, k - i, l - j, i + j + m)] += coef;
                ka = std::max(ka, k - i);
                kb = std::max(kb, l - j);
                kc = std::max(kc, i + j + m);
            }
    }
    if ((int)acc.size() > kMaxEdgeTerms || ka + kb + kc + 3 > kMaxRowEntries || kmax > 63) return;
    int n = 0;
    for (auto& kv : acc) {   // ordered by pattern
        if (kv.second >> 63) return;
        EdgeTerm& t = et->t[n++];
        t.pat = (uint8_t)std::get<0>(kv.first);
        t.a = (uint8_t)std::get<1>(kv.first);
        t.b = (uint8_t)std::get<2>(kv.first);
        t.c = (uint8_t)std::get<3>(kv.first);
        t.coef = (uint64_t)kv.second;
    }
    et->n = n;
    et->ka = ka; et->kb = kb; et->kc = kc;
    et->kmax = kmax;
}

// the Venn term table of a triangle / general-core pass (see VTerm): walk
// Listing 5's tree of every program on the host -- type by type, the next
// covering region with x > 0 fringes, s_r += x, coef *= C(s_r, x) (the
// multinomial split of region r built up one type at a time) -- and merge
// the leaves by (pattern, s).  Returns false (table off: per-program
// Listing 5 on the device) past the size limits or a 64-bit coefficient.
static bool build_venn_terms(const CoreProg& cp, std::vector<VTerm>* out, VennDev* hd) {
    const int q = cp.q, V = 1 << q;
    std::memset(hd, 0, sizeof *hd);
    out->clear();
    std::map<std::pair<int, std::vector<uint8_t>>, u128> acc;
    long long leaves = 0;
    const long long kLeafCap = 4000000;
    bool ok = true;
    int progs_per_pat[FSGC_MAXPATS] = {0};
    for (int pi = 0; pi < cp.nprog && ok; ++pi) {
        const FringeProg& fp = cp.prog[pi];
        ++progs_per_pat[fp.pat];
        std::vector<uint8_t> sv(V, 0);
        std::function<void(int, int, int, u128)> rec = [&](int t, int r0, int rem, u128 coef) {
            if (!ok) return;
            if (rem == 0) {
                if (t + 1 == fp.s || fp.s == 0) {
                    if (++leaves > kLeafCap) { ok = false; return; }
                    bool o = false;
                    u128& a = acc[std::make_pair((int)fp.pat, sv)];
                    a = add_ovf(a, coef, o);
                    if (o) ok = false;
                    return;
                }
                rec(t + 1, 1, fp.k[t + 1], coef);
                return;
            }
            const int A = fp.anch[t];
            for (int r = r0; r < V; ++r) {
                if ((r & A) != A) continue;
                for (int x = 1; x <= rem; ++x) {
                    sv[r] += (uint8_t)x;
                    bool o = false;
                    const u128 c = mul_ovf(coef, binom_ovf(sv[r], (uint32_t)x, o), o);
                    if (o) ok = false;
                    else rec(t, r + 1, rem - x, c);
                    sv[r] -= (uint8_t)x;
                }
            }
        };
        if (fp.s == 0) rec(0, 1, 0, 1);
        else rec(0, 1, fp.k[0], 1);
    }
    if (!ok || acc.empty() || (int)acc.size() > kMaxVennTerms) return false;
    int maxs[64] = {0};
    for (auto& kv : acc) {
        if (kv.second >> 64) return false;
        int nz = 0;
        for (int r = 1; r < V; ++r)
            if (kv.first.second[r]) { ++nz; maxs[r] = std::max(maxs[r], (int)kv.first.second[r]); }
        if (nz > kMaxVennNz) return false;
    }
    int nrows = 0;
    for (int r = 1; r < V; ++r) {
        if (maxs[r] > 63) return false;
        hd->maxs[r] = (uint8_t)maxs[r];
        hd->base[r] = (uint8_t)nrows;
        nrows += maxs[r];
    }
    if (nrows > kMaxVennRows) return false;
    for (auto& kv : acc) {
        VTerm t;
        std::memset(&t, 0, sizeof t);
        t.coef = (uint64_t)kv.second;
        t.pat = (uint8_t)kv.first.first;
        for (int r = 1; r < V; ++r)
            if (kv.first.second[r]) t.off[t.nz++] = (uint8_t)(hd->base[r] + kv.first.second[r] - 1);
        out->push_back(t);
    }
    int mp = 1;
    for (int i = 0; i < FSGC_MAXPATS; ++i) mp = std::max(mp, progs_per_pat[i]);
    hd->n = (int32_t)out->size();
    hd->nrows = nrows;
    hd->slack = std::log2((float)mp) + 2.f;
    return true;
}
// the Z-term table of a triangle-core pass (see ZTerm): false when some
// program is neither a single fringe type nor all-k = 1, or past the limits
static bool build_z_terms(const CoreProg& cp, const std::vector<std::vector<PartTerm>>& pterms,
                          std::vector<ZTerm>* out, VennDev* hd) {
    out->clear();
    if (cp.p != 3) return false;
    auto cmask = [&](int venn_mask) {
        int cm = 0;
        for (int b = 0; b < cp.q; ++b)
            if ((venn_mask >> b) & 1) cm |= 1 << cp.anchor_pos[b];
        return cm;
    };
    // (pattern, sorted factor list (cm << 8 | j)) -> coefficient
    std::map<std::pair<int, std::vector<int>>, int64_t> acc;
    int maxj[8] = {0}, zk = 0;
    for (int pi = 0; pi < cp.nprog; ++pi) {
        const FringeProg& fp = cp.prog[pi];
        zk = std::max(zk, (int)fp.ksum);
        if (fp.s == 0) {
            acc[std::make_pair((int)fp.pat, std::vector<int>())] += 1;
        } else if (fp.s == 1) {
            const int cm = cmask(fp.anch[0]), j = fp.k[0];
            if (j > 63) return false;
            maxj[cm] = std::max(maxj[cm], j);
            acc[std::make_pair((int)fp.pat, std::vector<int>{cm << 8 | j})] += 1;
        } else {
            if (pterms[pi].empty()) return false;
            for (const PartTerm& tm : pterms[pi]) {
                std::vector<int> f;
                for (int b = 0; b < tm.nb; ++b) {
                    const int cm = cmask(tm.mask[b]);
                    maxj[cm] = std::max(maxj[cm], 1);
                    f.push_back(cm << 8 | 1);
                }
                std::sort(f.begin(), f.end());
                acc[std::make_pair((int)fp.pat, f)] += tm.coef;
            }
        }
    }
    int nrows = 0;
    for (int cm = 1; cm < 8; ++cm) {
        hd->zmaxj[cm] = (uint8_t)maxj[cm];
        hd->zbase[cm] = (uint8_t)nrows;
        nrows += maxj[cm];
    }
    hd->zmaxj[0] = 0;
    for (auto& kv : acc) {
        if (kv.second == 0) continue;
        if (kv.first.second.size() > 6) return false;
        ZTerm t;
        std::memset(&t, 0, sizeof t);
        t.coef = kv.second;
        t.pat = (uint8_t)kv.first.first;
        for (int f : kv.first.second) {
            if ((f & 255) > 31) return false;
            t.f[t.nf++] = (uint8_t)((f >> 8) << 5 | (f & 255));
        }
        out->push_back(t);
    }
    if (out->empty() || (int)out->size() > kMaxZTerms || nrows > kMaxVennRows) return false;
    // per-pattern term ranges (the map orders the terms by pattern)
    for (int q = 0; q <= FSGC_MAXPATS; ++q) hd->zoff[q] = 0;
    for (const ZTerm& t : *out) hd->zoff[t.pat + 1]++;
    for (int q = 0; q < FSGC_MAXPATS; ++q) hd->zoff[q + 1] += hd->zoff[q];
    int progs_per_pat[FSGC_MAXPATS] = {0}, mp = 1;
    for (int pi = 0; pi < cp.nprog; ++pi) mp = std::max(mp, ++progs_per_pat[cp.prog[pi].pat]);
    hd->slack = std::log2((float)mp) + 2.f;
    // tier thresholds on the leaf's largest degree (the device compares
    // integers instead of evaluating the float bound per leaf)
    auto tier_max = [&](float lim) {
        int64_t lo = 0, hi = (int64_t)1 << 31;   // largest z with zk log2(z + 1) + slack < lim
        if ((float)zk * log2f(1.f) + hd->slack >= lim) return (int32_t)-1;
        while (hi - lo > 1) {
            const int64_t mid = (lo + hi) / 2;
            if ((float)zk * log2f((float)mid + 1.f) + hd->slack < lim) lo = mid; else hi = mid;
        }
        return (int32_t)std::min<int64_t>(lo, INT32_MAX);
    };
    hd->zmax64 = tier_max(55.f);
    hd->zmax128 = tier_max(119.f);
    // per pattern, the 64-bit tier of the row-free evaluation (arithmetic mod
    // 2^64 is exact when (i) every binomial factor C(Z, j) times j fits -- the
    // exact-division chain -- and (ii) the pattern's true per-leaf sum, which
    // is at most sum_programs prod_t C(Z_t, k_t) <= #programs prod_t Z^k_t / k_t!,
    // fits; partial sums and products may wrap, the ring arithmetic is exact
    // mod 2^64).  Both in log2 with a 2-bit margin, Z <= the leaf's max degree.
    {
        double lfact[64];
        lfact[0] = 0;
        for (int j = 1; j < 64; ++j) lfact[j] = lfact[j - 1] + std::log2((double)j);
        double nprog_p[FSGC_MAXPATS] = {0};
        for (int pi = 0; pi < cp.nprog; ++pi) nprog_p[cp.prog[pi].pat] += 1;
        for (int q = 0; q < FSGC_MAXPATS; ++q) {
            auto fits = [&](double lz) {   // lz = log2(Z + 1)
                double worst = 0;
                for (int pi = 0; pi < cp.nprog; ++pi) {
                    const FringeProg& fp = cp.prog[pi];
                    if (fp.pat != q) continue;
                    double b = 0;
                    for (int t = 0; t < fp.s; ++t) {
                        const int k = fp.k[t];
                        b += k * lz - lfact[k];
                        if (k * lz - lfact[k - 1] > 62.0) return false;   // C(Z, k) * k
                    }
                    worst = std::max(worst, b);
                }
                return worst + std::log2(std::max(1.0, nprog_p[q])) < 62.0;
            };
            int64_t lo = -1, hi = (int64_t)1 << 31;
            while (hi - lo > 1) {
                const int64_t mid = (lo + hi) / 2;
                if (fits(std::log2((double)mid + 1.0))) lo = mid; else hi = mid;
            }
            hd->zmax64p[q] = (int32_t)std::min<int64_t>(lo, INT32_MAX);
        }
    }
    hd->zn = (int32_t)out->size();
    hd->znrows = nrows;
    hd->zneed7 = maxj[7] > 0;
    hd->zk = zk;
    return true;
}
}  // namespace

// device copies of the partition-lattice term tables of a pattern batch;
// graph independent, so cached per (device, patterns) -- a new graph with the
// same patterns (e2e: load + count every step) allocates nothing here
struct DevTerms {
    PartTerm* terms = nullptr;
    int32_t* off = nullptr;
    int32_t* cnt = nullptr;
    VTerm* vterms = nullptr;        // Venn term tables of all passes
    ZTerm* zterms = nullptr;        // Z-term tables of all passes
    std::vector<VennDev> vhdr;      // per pass (terms point into vterms)
    ~DevTerms() {
        if (terms) cudaFree(terms);
        if (off) cudaFree(off);
        if (cnt) cudaFree(cnt);
        if (vterms) cudaFree(vterms);
        if (zterms) cudaFree(zterms);
    }
};

struct fsgc_plan {
    const fsgc_graph* g = nullptr;
    int npats = 0;
    std::vector<PassExec> passes;
    size_t ws_bytes = 0;
    int publish_mode = 1;
    int device = 0;
    // one per-edge support array c(e) = |N(u) & N(v)| for every pass that
    // reads it (edge, triangle and general cores), at ws[sup_off, + 4 m)
    int sup_first = -1;            // first pass reading it (-1: none)
    size_t sup_off = 0;            // the array; its work-queue counter 256 bytes before
    int64_t grid_sup = 1;          // merge kernel (small graphs / FSGC_SUP_MERGE_ONLY)
    int64_t grid_hash = 1;         // listing kernel, warp tables
    int64_t grid_hash_big = 1;     // listing kernel, block tables
    int hbits_big = 5;             // block tables: hash bits ...
    size_t smem_big = 0;           // ... and shared memory
    int sup_shard = 0, sup_nshards = 1;   // FSGC_FLAG_SHARD_SUPPORT: this shard's part
    std::vector<cudaEvent_t> ev;   // support begin/end, then begin/end per pass
    unsigned long long* trace = nullptr;
    std::shared_ptr<DevTerms> terms;   // partition-lattice terms of all programs
    ~fsgc_plan() {
        for (auto e : ev) cudaEventDestroy(e);
        if (trace) cudaFree(trace);
    }
};

extern "C" int fsgc_plan_create(const fsgc_graph* g, const fsgc_pattern* const* pats, int npats,
                                const fsgc_count_opts* opts_in, fsgc_plan** out) {
    if (!out) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_create: out is NULL");
    *out = nullptr;
    if (!g || !pats || npats < 1 || npats > FSGC_MAX_BATCH)
        FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_create: bad arguments");
    for (int i = 0; i < npats; ++i)
        if (!pats[i]) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_create: null pattern %d", i);
    fsgc_count_opts opts{0, -1, 0, 1, 0, 0};
    if (opts_in) opts = *opts_in;
    if (opts.shard_count < 1 || opts.shard_index < 0 || opts.shard_index >= opts.shard_count)
        FSGC_FAIL(FSGC_ERR_INVALID, "bad shard %d/%d", opts.shard_index, opts.shard_count);
    int dev = 0;
    FSGC_CUDA(cudaGetDevice(&dev));
    int rc = ensure_binom_table(dev);
    if (rc) return rc;
    std::vector<PassPlan> plans;
    rc = pass_plans(pats, npats, opts.no_symmetry_breaking, &plans);
    if (rc) return rc;

    std::unique_ptr<fsgc_plan> P(new fsgc_plan);
    P->g = g;
    P->npats = npats;
    P->device = dev;
    P->publish_mode = tune("FSGC_PUBLISH", 1);
    const int nsm = sm_count();
    size_t off = 0;
    for (const PassPlan& pp : plans) {
        PassExec X;
        X.plan = pp;
        const CoreProg& cp = pp.prog;
        const int64_t R = roots_for(g, cp.root_mode);
        int64_t b = opts.root_begin < 0 ? 0 : opts.root_begin;
        int64_t e = (opts.root_end < 0 || opts.root_end > R) ? R : opts.root_end;
        if (b > e) b = e;
        X.whole = opts.shard_count == 1 && opts.root_begin <= 0 && opts.root_end < 0;
        X.npc = np_class((int)pp.members.size());
        X.W = WorkDesc{b, e, opts.shard_index, opts.shard_count, 4,
                       (opts.flags & FSGC_FLAG_NO_DEGREE_FILTER) ? 0 : 1, nullptr};
        X.kind = cp.root_mode == ROOT_VERTEX ? 0 : (cp.p == 2 ? 1 : 2);
        // triangle cores with full symmetry breaking (u < v < w) over the
        // whole root range: the listing kernels (listing.cuh) enumerate them
        // by middle vertex; partial root ranges go to the generic kernel
        const bool whole_range = opts.root_begin <= 0 && opts.root_end < 0;
        if (X.kind == 2 && cp.p == 3 && cp.back[2] == 3 && cp.root_mode == ROOT_ORIENTED && (cp.gt[2] & 2) &&
            (cp.gt[2] & 1) && (cp.gt[1] & 1) && whole_range && !tune("FSGC_NO_TRI", 0)) {
            bool fits = true;   // Listing 5 stack bound of the triangle kernel
            for (int k = 0; k < cp.nprog; ++k) fits = fits && cp.prog[k].depth <= kTriStack;
            if (fits) X.kind = 3;
        }
        if (X.kind == 0) {
            X.W.chunk = 256;
            int64_t work = (e - b + opts.shard_count - 1) / opts.shard_count;
            X.grid = std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256,
                                                            (int64_t)nsm * occupancy(kernel_for(0, X.npc), 256, 0)));
        } else if (X.kind == 1) {
            int64_t mine = ((e - b) + 31) / 32;
            mine = (mine + opts.shard_count - 1) / opts.shard_count;
            build_edge_terms(cp, &X.et);
            if (tune("FSGC_NO_EDGE_TERMS", 0)) X.et.n = 0;
            X.smem_fc = X.et.n ? (size_t)(X.et.ka + X.et.kb + X.et.kc + 3) * 256 * sizeof(u128) : 0;
            X.grid = std::max<int64_t>(1, std::min<int64_t>((int64_t)nsm * occupancy(kernel_for(1, X.npc), 256, X.smem_fc),
                                                            (mine + 7) / 8));
            if (tune("FSGC_EDGE_BLOCKS", 0) > 0) X.grid = tune("FSGC_EDGE_BLOCKS", 0);
        } else if (X.kind == 3) {
            // grids and shared memory after the Venn tables (below); block
            // partials for both launches
            X.grid = (int64_t)nsm * 16;
        } else {
            X.smem = (size_t)kCoreWarps * (32 * FSGC_MAXC + 32 * (1u << cp.q)) * sizeof(uint32_t);
            int64_t nchunks = ((e - b) + X.W.chunk - 1) / X.W.chunk;
            int64_t mine = (nchunks + opts.shard_count - 1) / opts.shard_count;
            X.grid = std::max<int64_t>(1, std::min<int64_t>((int64_t)nsm * occupancy(kernel_for(2, X.npc), kCoreWarps * 32, X.smem),
                                                            (mine + kCoreWarps - 1) / kCoreWarps));
        }
        X.uses_sup = X.kind != 0 && g->m > 0;
        if (X.uses_sup && P->sup_first < 0) P->sup_first = (int)P->passes.size();
        X.bytes = ((size_t)X.grid * sizeof(BlockPartial) + 255) & ~(size_t)255;   // block partials
        P->passes.push_back(X);
    }
    // workspace: [pass headers][support queue counters (256 B)][support
    // array][pass block partials] -- the zeroed part is one contiguous range
    const size_t np_ = P->passes.size();
    P->sup_off = np_ * kHdrBytes + 256;
    off = P->sup_off + (P->sup_first >= 0 ? (((size_t)g->m * sizeof(int) + 255) & ~(size_t)255) : 0);
    for (size_t i = 0; i < np_; ++i) {
        PassExec& X = P->passes[i];
        X.ws_off = i * kHdrBytes;
        X.parts_off = off - X.ws_off;
        off += X.bytes;
    }
    if (P->sup_first >= 0) {
        if (g->sup_hash) {
            typedef WarpTabLayout<0> LS;
            P->grid_hash = std::max<int64_t>(1, std::min<int64_t>(
                (int64_t)nsm * occupancy((const void*)list_warp_kernel<0, 1>, kWarpTabWarps * 32, LS::bytes),
                (g->nsup_units + kWarpTabWarps - 1) / kWarpTabWarps));
            P->hbits_big = table_hbits(g->sup_maxout);
            P->smem_big = blocktab_table_bytes(1 << P->hbits_big, (int)g->sup_maxout, false);
            const int occ = occupancy((const void*)list_block_kernel<0, 1>, kBlockTabWarps * 32, P->smem_big);
            if (g->nsup_units_big > 0 && occ == 0)
                FSGC_FAIL(FSGC_ERR_INVALID, "block table of out-degree %lld does not fit shared memory",
                          (long long)g->sup_maxout);
            P->grid_hash_big = std::max<int64_t>(1, std::min<int64_t>((int64_t)nsm * occ, g->nsup_units_big));
        }
        if (g->nsup_merge > 0)
            P->grid_sup = std::max<int64_t>(1, std::min<int64_t>(
                (int64_t)nsm * occupancy((const void*)support_kernel, 256, 0), (g->nsup_merge + 255) / 256));
        if ((opts.flags & FSGC_FLAG_SHARD_SUPPORT) && opts.shard_count > 1) {
            P->sup_shard = opts.shard_index;
            P->sup_nshards = opts.shard_count;
        }
    }
    P->ws_bytes = off;
    {   // partition-lattice term tables -> device (cached)
        static std::mutex tmu;
        static std::map<std::vector<uint64_t>, std::shared_ptr<DevTerms>> tcache;
        std::vector<uint64_t> tkey{(uint64_t)dev, (uint64_t)opts.no_symmetry_breaking};
        for (int i = 0; i < npats; ++i) tkey.push_back(pats[i]->uid);
        std::lock_guard<std::mutex> lock(tmu);
        auto it = tcache.find(tkey);
        std::vector<PartTerm> all;
        std::vector<int32_t> offs, cnts;
        for (auto& X : P->passes) {
            X.term_base = (int)offs.size();
            for (int k = 0; k < X.plan.prog.nprog; ++k) {
                const auto& T = X.plan.terms[k];
                offs.push_back((int32_t)all.size());
                cnts.push_back(T.empty() ? -1 : (int32_t)T.size());
                all.insert(all.end(), T.begin(), T.end());
            }
        }
        if (it != tcache.end()) {
            P->terms = it->second;
        } else {
            if (all.empty()) all.push_back(PartTerm{});
            if (offs.empty()) { offs.push_back(0); cnts.push_back(-1); }
            std::shared_ptr<DevTerms> T(new DevTerms);
            FSGC_CUDA(cudaMalloc(&T->terms, all.size() * sizeof(PartTerm)));
            FSGC_CUDA(cudaMalloc(&T->off, offs.size() * sizeof(int32_t)));
            FSGC_CUDA(cudaMalloc(&T->cnt, cnts.size() * sizeof(int32_t)));
            FSGC_CUDA(cudaMemcpy(T->terms, all.data(), all.size() * sizeof(PartTerm), cudaMemcpyHostToDevice));
            FSGC_CUDA(cudaMemcpy(T->off, offs.data(), offs.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
            FSGC_CUDA(cudaMemcpy(T->cnt, cnts.data(), cnts.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
            // Venn term tables (pattern-only, so cached with the rest)
            std::vector<VTerm> vall;
            std::vector<size_t> vbase;
            std::vector<ZTerm> zall;
            std::vector<size_t> zbase;
            for (auto& X : P->passes) {
                VennDev hd;
                std::memset(&hd, 0, sizeof hd);
                std::vector<VTerm> vt;
                if ((X.kind == 2 || X.kind == 3) && !tune("FSGC_NO_VENN_TERMS", 0) &&
                    build_venn_terms(X.plan.prog, &vt, &hd)) {
                    vbase.push_back(vall.size());
                    vall.insert(vall.end(), vt.begin(), vt.end());
                } else {
                    std::memset(&hd, 0, sizeof hd);
                    vbase.push_back(0);
                }
                // triangle cores: the Z-term table when every program allows it
                std::vector<ZTerm> zt;
                VennDev zh;
                std::memset(&zh, 0, sizeof zh);
                if (X.kind == 3 && !tune("FSGC_NO_Z_TERMS", 0) && build_z_terms(X.plan.prog, X.plan.terms, &zt, &zh)) {
                    zbase.push_back(zall.size());
                    zall.insert(zall.end(), zt.begin(), zt.end());
                    hd.zn = zh.zn; hd.znrows = zh.znrows; hd.zneed7 = zh.zneed7; hd.zk = zh.zk;
                    hd.slack = std::max(hd.slack, zh.slack);
                    std::memcpy(hd.zmaxj, zh.zmaxj, 8);
                    std::memcpy(hd.zbase, zh.zbase, 8);
                    std::memcpy(hd.zoff, zh.zoff, sizeof hd.zoff);
                    hd.zmax64 = zh.zmax64;
                    std::memcpy(hd.zmax64p, zh.zmax64p, sizeof hd.zmax64p);
                    hd.zmax128 = zh.zmax128;
                } else {
                    zbase.push_back(0);
                }
                T->vhdr.push_back(hd);
            }
            if (!zall.empty()) {
                FSGC_CUDA(cudaMalloc(&T->zterms, zall.size() * sizeof(ZTerm)));
                FSGC_CUDA(cudaMemcpy(T->zterms, zall.data(), zall.size() * sizeof(ZTerm), cudaMemcpyHostToDevice));
            }
            for (size_t i = 0; i < T->vhdr.size(); ++i)
                if (T->vhdr[i].zn) T->vhdr[i].zterms = T->zterms + zbase[i];
            if (!vall.empty()) {
                FSGC_CUDA(cudaMalloc(&T->vterms, vall.size() * sizeof(VTerm)));
                FSGC_CUDA(cudaMemcpy(T->vterms, vall.data(), vall.size() * sizeof(VTerm), cudaMemcpyHostToDevice));
            }
            for (size_t i = 0; i < T->vhdr.size(); ++i)
                if (T->vhdr[i].n) T->vhdr[i].terms = T->vterms + vbase[i];
            if (tcache.size() > 256) tcache.clear();
            tcache[tkey] = T;
            P->terms = T;
        }
        // Venn tables -> passes: rows in dynamic shared memory, grids re-sized
        for (size_t i = 0; i < P->passes.size(); ++i) {
            PassExec& X = P->passes[i];
            X.vd = P->terms->vhdr[i];
            if (!X.vd.n) continue;
            // small tables: a diagram per lane, rows per thread in dynamic
            // shared memory; large ones (more than 48 KB of rows per block or
            // FSGC_VENN_WARP_TERMS terms): a diagram per warp, rows per warp
            const int threads = X.kind == 3 ? kTriWarps * 32 : kCoreWarps * 32;
            const size_t lane_rows = (size_t)X.vd.nrows * sizeof(u128) * threads;
            X.vd.warp = (lane_rows > 48 * 1024 || X.vd.n >= tune("FSGC_VENN_WARP_TERMS", 1024)) ? 1 : 0;
            X.smem_vd = X.vd.warp ? 0 : lane_rows;
            if (!X.vd.warp) {
                const int64_t per = (int64_t)nsm * occupancy(kernel_for(X.kind, X.npc), threads, X.smem + X.smem_vd);
                X.grid = std::max<int64_t>(1, std::min<int64_t>(X.grid, per));
            }
            if (tune("FSGC_VENN_INFO", 0))
                fprintf(stderr, "[venn] pass kind %d: %d terms, %d rows, %s mode; z-terms %d (%d rows, k %d)\n",
                        X.kind, X.vd.n, X.vd.nrows, X.vd.warp ? "warp" : "lane", X.vd.zn, X.vd.znrows, X.vd.zk);
        }
        // triangle-core passes: the two listing launches (warp tables, block
        // tables), persistent grids at full occupancy
        for (auto& X : P->passes) {
            if (X.kind != 3) continue;
            // lane-mode term rows (kTriWarps * 32 threads): Venn table and/or Z table
            // (the Z-term path keeps no rows: binomials are computed per factor)
            const size_t rows = X.vd.zn ? (size_t)0 : X.smem_vd;
            // Z-term-only kernels when the tier bound of the largest possible
            // leaf (max degree) stays below the 128-bit limit of tri_flush
            X.zonly = X.vd.zn > 0 && !tune("FSGC_NO_ZONLY", 0) && g->max_degree <= X.vd.zmax128;
            X.smem = (X.zonly ? WarpTabLayout<2>::bytes : WarpTabLayout<1>::bytes) + rows;
            int occ = occupancy(tri_kernel(X.zonly, false, X.npc), kWarpTabWarps * 32, X.smem);
            if (occ == 0) FSGC_FAIL(FSGC_ERR_INVALID, "triangle-core pass: shared memory %zu B does not fit", X.smem);
            const int64_t units_w = (g->nsup_units + opts.shard_count - 1) / opts.shard_count;
            const int64_t units_b = (g->nsup_units_big + opts.shard_count - 1) / opts.shard_count;
            X.grid = std::max<int64_t>(1, std::min<int64_t>((int64_t)nsm * std::min(occ, 16),
                                                            (units_w + kWarpTabWarps - 1) / kWarpTabWarps));
            X.hbits2 = table_hbits(g->sup_maxout);
            // block tables: warps per block with the most resident warps
            // (Z-only kernel: 8 or 12 -- a large table fits twice per SM
            // with 12 warps each; MODE 1: 8)
            {
                int best = -1;
                for (int nw : X.zonly ? std::vector<int>{8, 12} : std::vector<int>{kBlockTriWarps}) {
                    const size_t sm2 = blocktab_table_bytes(1 << X.hbits2, (int)g->sup_maxout, true) +
                                       nw * blocktab_warp_bytes(X.zonly ? 2 : 1) + rows;
                    const int o = occupancy(tri_kernel(X.zonly, true, X.npc), nw * 32, sm2);
                    if (o * nw > best) { best = o * nw; X.nwb2 = nw; X.smem2 = sm2; occ = o; }
                }
            }
            if (occ == 0 && units_b > 0)
                FSGC_FAIL(FSGC_ERR_INVALID, "triangle-core pass: block table of out-degree %lld does not fit "
                          "shared memory (%zu B)", (long long)g->sup_maxout, X.smem2);
            X.grid2 = std::max<int64_t>(1, std::min<int64_t>((int64_t)nsm * std::max(1, std::min(occ, 16)) ,
                                                             std::max<int64_t>(1, units_b)));
            if (tune("FSGC_VENN_INFO", 0))
                fprintf(stderr, "[tri] zonly %d; warp tables: %zu B smem, grid %lld; block tables (max out %lld): "
                        "%d warps, %zu B smem, %d blocks/SM, grid %lld\n", (int)X.zonly, X.smem, (long long)X.grid,
                        (long long)g->sup_maxout, X.nwb2, X.smem2, occ, (long long)X.grid2);
            if (X.grid + X.grid2 > (int64_t)nsm * 16)
                FSGC_FAIL(FSGC_ERR_INTERNAL, "triangle-core pass: block partials overflow");
        }
    }
    P->ev.resize(2 + 2 * P->passes.size());
    for (auto& ev : P->ev) FSGC_CUDA(cudaEventCreate(&ev));
    if (tune("FSGC_TRACE", 0)) {
        FSGC_CUDA(cudaMalloc(&P->trace, (size_t)2 * 1024 * 1024));
        FSGC_CUDA(cudaMemset(P->trace, 0, (size_t)2 * 1024 * 1024));
    }
    *out = P.release();
    return FSGC_OK;
}

extern "C" int fsgc_plan_workspace_bytes(const fsgc_plan* P, size_t* ws, size_t* raw) {
    if (!P) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_workspace_bytes: null plan");
    if (ws) *ws = P->ws_bytes;
    if (raw) *raw = kRawPassBytes * P->passes.size();
    return FSGC_OK;
}

extern "C" int fsgc_plan_support_region(const fsgc_plan* P, size_t* offset, int64_t* count) {
    if (!P || !offset || !count) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_support_region: null argument");
    *offset = P->sup_off;
    *count = P->sup_first >= 0 ? P->g->m : 0;
    return FSGC_OK;
}

extern "C" int fsgc_plan_enqueue_stage(const fsgc_plan* P, void* workspace, void* raw_out, int stages,
                                       void* stream_) {
    if (!P || !workspace || !raw_out) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_enqueue: null argument");
    if (stages & ~FSGC_STAGE_ALL) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_enqueue_stage: bad stage mask %d", stages);
    cudaStream_t st = (cudaStream_t)stream_;
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    FSGC_CUDA(cudaStreamIsCapturing(st, &cap));
    // inside a graph capture the timing events must be "external" records
    const unsigned evflags = cap == cudaStreamCaptureStatusActive ? cudaEventRecordExternal : 0;
    const fsgc_graph* g = P->g;
    GraphDev G{g->offsets, g->adj, g->row, g->osrc, g->odst};
    OrientDev O{g->split, g->oofs};
    int* dsup = (int*)((unsigned char*)workspace + P->sup_off);
    const size_t np_ = P->passes.size();
    const size_t sup_bytes = P->sup_first >= 0 ? (size_t)g->m * sizeof(int) : 0;
    // zero the headers (count stage) and the queue + support array (support
    // stage): one memset when both stages run
    if ((stages & FSGC_STAGE_ALL) == FSGC_STAGE_ALL)
        FSGC_CUDA(cudaMemsetAsync(workspace, 0, P->sup_off + sup_bytes, st));
    else if (stages & FSGC_STAGE_COUNT)
        FSGC_CUDA(cudaMemsetAsync(workspace, 0, np_ * kHdrBytes, st));
    else
        FSGC_CUDA(cudaMemsetAsync((unsigned char*)workspace + np_ * kHdrBytes, 0, 256 + sup_bytes, st));
    if ((stages & FSGC_STAGE_SUPPORT) && P->sup_first >= 0) {   // (A) per-edge common-neighbour counts
        unsigned long long* dq = (unsigned long long*)((unsigned char*)dsup - 256);   // 2 queue counters
        unsigned long long* dq1 = dq + 1;
        FSGC_CUDA(cudaEventRecordWithFlags(P->ev[0], st, evflags));
        // listing kernels (graphs >= FSGC_SUP_HASH_MIN_M edges), else the
        // merge kernel over every oriented edge (also FSGC_SUP_MERGE_ONLY=1:
        // the independent check of the listing kernels)
        const bool merge_only = g->nsup_merge > 0 && (!g->sup_hash || tune("FSGC_SUP_MERGE_ONLY", 0) != 0);
        HubDev Hd{g->hub_base, g->hub_words, g->hub_bits};
        const CoreProg* cp0 = &P->passes[P->sup_first].plan.prog;   // unused by the support visitor
        WorkDesc W0{};
        VennDev V0{};
        Sink S0{};
        if (!merge_only && g->nsup_units_big > 0) {
            int hb = P->hbits_big, mo = (int)g->sup_maxout;
            void* args[] = {(void*)&G, (void*)&O, (void*)&Hd, (void*)&g->rev, (void*)&g->sup_units_big,
                            (void*)&g->nsup_units_big, (void*)&hb, (void*)&mo, (void*)&dsup, (void*)&dq1,
                            (void*)&P->sup_shard, (void*)&P->sup_nshards, (void*)cp0, (void*)&W0, (void*)&V0,
                            (void*)&S0};
            FSGC_CUDA(cudaLaunchKernel((const void*)list_block_kernel<0, 1>, dim3((unsigned)P->grid_hash_big),
                                       dim3(kBlockTabWarps * 32), args, P->smem_big, st));
        }
        if (!merge_only && g->nsup_units > 0) {
            void* args[] = {(void*)&G, (void*)&O, (void*)&Hd, (void*)&g->rev, (void*)&g->sup_units,
                            (void*)&g->nsup_units, (void*)&dsup, (void*)&dq, (void*)&P->sup_shard,
                            (void*)&P->sup_nshards, (void*)cp0, (void*)&W0, (void*)&V0, (void*)&S0};
            FSGC_CUDA(cudaLaunchKernel((const void*)list_warp_kernel<0, 1>, dim3((unsigned)P->grid_hash),
                                       dim3(kWarpTabWarps * 32), args, WarpTabLayout<0>::bytes, st));
        }
        if (merge_only) {
            support_kernel<<<(int)P->grid_sup, 256, 0, st>>>(G, O, g->nsup_merge, dsup, g->sorder, g->ssrc, g->sdst,
                                                             P->sup_shard, P->sup_nshards,
                                                             P->trace ? P->trace + (1 << 17) : nullptr);
            FSGC_CUDA(cudaGetLastError());
        }
        FSGC_CUDA(cudaEventRecordWithFlags(P->ev[1], st, evflags));
    }
    if (!(stages & FSGC_STAGE_COUNT)) return FSGC_OK;
    for (size_t pi = 0; pi < P->passes.size(); ++pi) {
        const PassExec& X = P->passes[pi];
        unsigned char* base = (unsigned char*)workspace + X.ws_off;
        AccDev* dacc = (AccDev*)base;
        unsigned long long* dmatch = (unsigned long long*)(base + sizeof(AccDev) * FSGC_MAXPATS);
        unsigned long long* dqueue = dmatch + 1;
        unsigned int* dticket = (unsigned int*)(dmatch + 3);
        Sink S{dacc, dmatch, (BlockPartial*)(base + X.parts_off), dticket, P->publish_mode};
        WorkDesc W = X.W;
        const CoreProg& cp = X.plan.prog;
        FSGC_CUDA(cudaEventRecordWithFlags(P->ev[2 + 2 * pi], st, evflags));
        if (W.end > W.begin) {
            const void* fn = kernel_for(X.kind, X.npc);
            void* args_v[] = {(void*)&G, (void*)&cp, (void*)&W, (void*)&S};
            void* args_e[] = {(void*)&G, (void*)&O, (void*)&cp, (void*)&W, (void*)&dsup, (void*)&X.et, (void*)&S};
            HubDev Hd{g->hub_base, g->hub_words, g->hub_bits};
            TermDev TD{P->terms->terms, P->terms->off + X.term_base, P->terms->cnt + X.term_base};
            void* args_c[] = {(void*)&G, (void*)&O, (void*)&Hd, (void*)&cp, (void*)&W, (void*)&dsup, (void*)&TD,
                              (void*)&X.vd, (void*)&S, (void*)&dqueue};
            // triangle cores: two listing launches into one sink (one 128-bit
            // atomic per block; the block launch's partials after the warp
            // launch's), queues at dmatch[1], dmatch[2]
            Sink St = S;
            St.mode = 1;
            Sink St2 = St;
            St2.parts = St.parts + X.grid;
            unsigned long long* dqueue2 = dmatch + 2;
            int shard = W.shard, nsh = W.nshards, hb2 = X.hbits2, mo = (int)g->sup_maxout;
            void* args_t[] = {(void*)&G, (void*)&O, (void*)&Hd, (void*)&g->rev, (void*)&g->sup_units,
                              (void*)&g->nsup_units, (void*)&dsup, (void*)&dqueue, (void*)&shard, (void*)&nsh,
                              (void*)&cp, (void*)&W, (void*)&X.vd, (void*)&St};
            void* args_t2[] = {(void*)&G, (void*)&O, (void*)&Hd, (void*)&g->rev, (void*)&g->sup_units_big,
                               (void*)&g->nsup_units_big, (void*)&hb2, (void*)&mo, (void*)&dsup, (void*)&dqueue2,
                               (void*)&shard, (void*)&nsh, (void*)&cp, (void*)&W, (void*)&X.vd, (void*)&St2};
            if (X.kind == 0)
                FSGC_CUDA(cudaLaunchKernel(fn, dim3((unsigned)X.grid), dim3(256), args_v, 0, st));
            else if (X.kind == 1)    // (B) fringe counts per root edge
                FSGC_CUDA(cudaLaunchKernel(fn, dim3((unsigned)X.grid), dim3(256), args_e, X.smem_fc, st));
            else if (X.kind == 3) {
                if (g->nsup_units_big > 0)
                    FSGC_CUDA(cudaLaunchKernel(tri_kernel(X.zonly, true, X.npc), dim3((unsigned)X.grid2),
                                               dim3(X.nwb2 * 32), args_t2, X.smem2, st));
                if (g->nsup_units > 0)
                    FSGC_CUDA(cudaLaunchKernel(tri_kernel(X.zonly, false, X.npc), dim3((unsigned)X.grid),
                                               dim3(kWarpTabWarps * 32), args_t, X.smem, st));
            }
            else
                FSGC_CUDA(cudaLaunchKernel(fn, dim3((unsigned)X.grid), dim3(kCoreWarps * 32), args_c,
                                           X.smem + X.smem_vd, st));
        }
        FSGC_CUDA(cudaEventRecordWithFlags(P->ev[3 + 2 * pi], st, evflags));
    }
    // every pass's raw sums in one strided copy (header pitch -> raw pitch)
    FSGC_CUDA(cudaMemcpy2DAsync(raw_out, kRawPassBytes, workspace, kHdrBytes, kRawPassBytes - 8, np_,
                                cudaMemcpyDefault, st));
    return FSGC_OK;
}

extern "C" int fsgc_plan_enqueue(const fsgc_plan* P, void* workspace, void* raw_out, void* stream_) {
    if (P && P->sup_nshards > 1)
        FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_enqueue: a plan with a sharded support pass runs in two "
                                    "stages (fsgc_plan_enqueue_stage) with the support sum in between");
    return fsgc_plan_enqueue_stage(P, workspace, raw_out, FSGC_STAGE_ALL, stream_);
}

extern "C" int fsgc_plan_decode(const fsgc_plan* P, const void* raw, fsgc_result* results) {
    if (!P || !raw || !results) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_plan_decode: null argument");
    std::memset(results, 0, sizeof(fsgc_result) * P->npats);
    for (size_t pi = 0; pi < P->passes.size(); ++pi) {
        const PassExec& X = P->passes[pi];
        const AccDev* acc = (const AccDev*)((const unsigned char*)raw + pi * kRawPassBytes);
        unsigned long long matches;
        std::memcpy(&matches, (const unsigned char*)raw + pi * kRawPassBytes + sizeof(AccDev) * FSGC_MAXPATS, 8);
        // the shared support pass is reported with the first pass reading it
        const bool sup_here = (int)pi == P->sup_first;
        float kms = 0.f, ams = 0.f;
        if (sup_here && cudaEventElapsedTime(&ams, P->ev[0], P->ev[1]) != cudaSuccess) ams = -1.f;
        if (cudaEventElapsedTime(&kms, P->ev[2 + 2 * pi], P->ev[3 + 2 * pi]) != cudaSuccess) kms = -1.f;
        cudaGetLastError();   // timing is best effort (e.g. events recorded inside a graph)
        const fsgc_graph* g = P->g;
        const bool merge_only = g->nsup_merge > 0 && (!g->sup_hash || tune("FSGC_SUP_MERGE_ONLY", 0) != 0);
        const int sup_launches = merge_only ? 1 : (g->nsup_units > 0 ? 1 : 0) + (g->nsup_units_big > 0 ? 1 : 0);
        const int pass_launches = X.W.end <= X.W.begin ? 0
                                  : X.kind == 3 ? (g->nsup_units > 0 ? 1 : 0) + (g->nsup_units_big > 0 ? 1 : 0)
                                                : 1;
        const int launches = pass_launches + (sup_here ? sup_launches : 0);
        for (size_t mi = 0; mi < X.plan.members.size(); ++mi) {
            fsgc_result& r = results[X.plan.members[mi]];
            r.raw.lo = acc[mi].lo;
            r.raw.hi = acc[mi].hi;
            r.overflow = acc[mi].ovf ? 1 : 0;
            r.divisor = X.plan.divisor[mi];
            r.core_matches = matches;
            r.root_pattern_vertex = X.plan.root_pattern_vertex[mi];
            r.kernel_ms = kms;
            r.aux_ms = ams;
            r.kernel_launches = launches;
            r.pass_index = (int32_t)pi;
            r.pass_kind = X.kind;
            if (X.whole) {
                int rc = fsgc_finalize(r.raw, r.divisor, r.overflow, &r.count, &r.overflow);
                if (rc) return rc;
            }
        }
        if (P->trace && X.kind == 1) {
            std::vector<unsigned long long> all((size_t)2 * 1024 * 1024 / 8);
            FSGC_CUDA(cudaMemcpy(all.data(), P->trace, all.size() * 8, cudaMemcpyDeviceToHost));
            for (int part = 0; part < 2; ++part) {
                const unsigned long long* h = all.data() + (part ? (1 << 17) : 0);
                unsigned long long t0 = ~0ull, t1 = 0;
                std::vector<std::pair<unsigned long long, int>> d;
                for (size_t w = 0; w < (1 << 14); ++w) {
                    if (!h[8 * w]) continue;
                    t0 = std::min(t0, h[8 * w]);
                    t1 = std::max(t1, h[8 * w + 1]);
                    d.push_back({h[8 * w + 1] - h[8 * w], (int)w});
                }
                std::sort(d.rbegin(), d.rend());
                fprintf(stderr, "[trace %s] warps=%zu span=%.1fus; slowest:", part ? "support" : "fc", d.size(),
                        (t1 - t0) / 1e3);
                for (size_t i = 0; i < std::min<size_t>(4, d.size()); ++i) {
                    int w = d[i].second;
                    const unsigned long long* r = h + 8 * w;
                    fprintf(stderr, " w%d(sm%llu,ch%llu,start+%.1f,%.1fus", w, r[2], r[3], (r[0] - t0) / 1e3,
                            d[i].first / 1e3);
                    if (r[4]) fprintf(stderr, " ld1 %.1f ld2 %.1f fc %.1f pub %.1f", (r[4] - r[0]) / 1e3,
                                      (r[5] - r[4]) / 1e3, (r[6] - r[5]) / 1e3, (r[1] - r[6]) / 1e3);
                    fprintf(stderr, ")");
                }
                fprintf(stderr, "\n");
            }
            cudaMemset(P->trace, 0, (size_t)2 * 1024 * 1024);
        }
    }
    return FSGC_OK;
}

extern "C" void fsgc_plan_free(fsgc_plan* P) { delete P; }

// ---------------------------------------------------------------- fsgc_count
// Convenience path: cached plan + per-thread workspace / pinned result
// buffers, enqueue, synchronise, decode.
namespace {
struct ThreadBuffers {
    void* ws = nullptr;
    size_t ws_size = 0;
    int ws_dev = -1;
    void* raw = nullptr;
    size_t raw_size = 0;
    ~ThreadBuffers() {
        if (ws) cudaFree(ws);
        if (raw) cudaFreeHost(raw);
    }
};
}  // namespace

extern "C" int fsgc_count(const fsgc_graph* g, const fsgc_pattern* const* pats, int npats,
                          const fsgc_count_opts* opts_in, fsgc_result* results, void* stream_) {
    if (!g || !pats || !results || npats < 1 || npats > FSGC_MAX_BATCH)
        FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_count: bad arguments");
    for (int i = 0; i < npats; ++i)
        if (!pats[i]) FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_count: null pattern %d", i);
    fsgc_count_opts opts{0, -1, 0, 1, 0, 0};
    if (opts_in) opts = *opts_in;
    cudaStream_t st = (cudaStream_t)stream_;

    // plan cache: graph identity + pattern uids + options
    std::vector<uint64_t> key{g->uid, (uint64_t)opts.root_begin, (uint64_t)opts.root_end,
                              (uint64_t)opts.shard_index, (uint64_t)opts.shard_count,
                              (uint64_t)opts.no_symmetry_breaking, (uint64_t)opts.flags};
    for (int i = 0; i < npats; ++i) key.push_back(pats[i]->uid);
    static std::mutex mu;
    static std::map<std::vector<uint64_t>, std::shared_ptr<fsgc_plan>> cache;
    std::shared_ptr<fsgc_plan> plan;
    {
        std::lock_guard<std::mutex> lock(mu);
        auto it = cache.find(key);
        if (it != cache.end()) plan = it->second;
    }
    if (!plan) {
        fsgc_plan* p = nullptr;
        int rc = fsgc_plan_create(g, pats, npats, &opts, &p);
        if (rc) return rc;
        plan.reset(p, fsgc_plan_free);
        std::lock_guard<std::mutex> lock(mu);
        if (cache.size() > 256) cache.clear();
        cache[key] = plan;
    }
    static thread_local ThreadBuffers tb;
    size_t wsb = 0, rawb = 0;
    fsgc_plan_workspace_bytes(plan.get(), &wsb, &rawb);
    if (tb.ws_size < wsb || tb.ws_dev != plan->device) {
        if (tb.ws) cudaFree(tb.ws);
        tb.ws = nullptr;
        tb.ws_size = 0;
        FSGC_CUDA(cudaMalloc(&tb.ws, std::max<size_t>(wsb, 1 << 20)));
        tb.ws_size = std::max<size_t>(wsb, 1 << 20);
        tb.ws_dev = plan->device;
    }
    if (tb.raw_size < rawb) {
        if (tb.raw) cudaFreeHost(tb.raw);
        tb.raw = nullptr;
        FSGC_CUDA(cudaMallocHost(&tb.raw, std::max<size_t>(rawb, 4096)));
        tb.raw_size = std::max<size_t>(rawb, 4096);
    }
    if (plan->sup_nshards > 1)
        FSGC_FAIL(FSGC_ERR_INVALID, "fsgc_count: FSGC_FLAG_SHARD_SUPPORT needs the staged plan API "
                                    "(the shards' support arrays are summed between the stages)");
    int rc = fsgc_plan_enqueue(plan.get(), tb.ws, tb.raw, st);
    if (rc) return rc;
    FSGC_CUDA(cudaStreamSynchronize(st));
    return fsgc_plan_decode(plan.get(), tb.raw, results);
}
