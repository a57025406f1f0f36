// count_dev.cuh -- device side of fsgc_count (types, kernels, fc arithmetic).
// Included by count.cu (host side: plans, launches; support kernels) and by
// count_np.cu, compiled once per accumulator class NP in {1,2,4,8,16} so the
// kernel instantiations build in parallel.  Everything here sits in an
// anonymous namespace: each translation unit has its own copies of the
// kernels and of the constant tables (dev_consts_init fills them).
//
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
#pragma once
#include "devbuf.cuh"
#include "u128.cuh"
#include "fc.cuh"

#define FULLMASK 0xffffffffu

namespace {

// Pascal's triangle, one thread per k column walking n (mod 2^64)
__global__ void binom_table_init() {
    const int k = threadIdx.x;
    if (k >= kBinomK) return;
    // C(n, k) = C(n-1, k) + C(n-1, k-1): do it row-serially in one warp
    __shared__ uint64_t row[kBinomK];
    for (int n = 0; n < kBinomN; ++n) {
        uint64_t v;
        if (k == 0) v = 1;
        else if (n == 0) v = 0;
        else v = row[k] + row[k - 1];
        __syncwarp();
        row[k] = v;
        g_binom[n][k] = v;
        __syncwarp();
    }
}



struct GraphDev {
    const int64_t* __restrict__ offs;
    const int32_t* __restrict__ adj;
    const int32_t* __restrict__ row;
    const int32_t* __restrict__ osrc;
    const int32_t* __restrict__ odst;
};

struct WorkDesc {
    int64_t begin, end;   // root item range
    int32_t shard, nshards;
    int32_t chunk;        // items per queue grab
    int32_t degfilter;    // 1: apply the degree filter
    unsigned long long* trace;  // optional per-warp (start, end, smid, chunks) timing
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

struct AccDev {
    unsigned long long lo, hi;
    unsigned int ovf, pad;
    unsigned long long pad2;
};

__device__ __forceinline__ bool contains(const int32_t* __restrict__ L, int len, int x) {
    int lo = 0, hi = len;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(L + mid) < x) lo = mid + 1; else hi = mid;
    }
    return lo < len && __ldg(L + lo) == x;
}

// first index with L[i] > x
__device__ __forceinline__ int upper_bound(const int32_t* __restrict__ L, int len, int x) {
    int lo = 0, hi = len;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (__ldg(L + mid) <= x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ void warp_reduce_u128(u128& v, bool& ovf) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        uint64_t lo = __shfl_down_sync(FULLMASK, u128_lo(v), o);
        uint64_t hi = __shfl_down_sync(FULLMASK, u128_hi(v), o);
        int f = __shfl_down_sync(FULLMASK, (int)ovf, o);
        v = add_ovf(v, u128_make(lo, hi), ovf);
        ovf |= (f != 0);
    }
}

__device__ __forceinline__ void atomic_add_u128(AccDev* a, u128 v, bool ovf) {
    const uint64_t lo = u128_lo(v), hi = u128_hi(v);
    bool o = ovf;
    uint64_t carry = 0;
    if (lo) {
        unsigned long long old = atomicAdd(&a->lo, (unsigned long long)lo);
        carry = (old + lo < old) ? 1 : 0;
    }
    uint64_t hadd = hi + carry;
    if (hadd < hi) o = true;
    if (hadd) {
        unsigned long long oldh = atomicAdd(&a->hi, (unsigned long long)hadd);
        if (oldh + hadd < oldh) o = true;
    }
    if (o) atomicOr(&a->ovf, 1u);
}

// One warp's pattern accumulators in SHARED memory (the triangle-core listing
// kernels keep no per-lane register accumulators across the listing); lanes
// may add concurrently, so the 128-bit add is two 64-bit atomics with carry.
struct SAcc {
    AccDev* a;   // [patterns]
    __device__ __forceinline__ void add(int pat, u128 c, bool o) const {
        if (c != 0 || o) atomic_add_u128(a + pat, c, o);
    }
};

// Per-lane accumulators for NP patterns, register resident (pattern index
// resolved by an unrolled compare, never by dynamic indexing).
template <int NP>
struct AccN {
    u128 v[NP];
    uint32_t ovf;
    __device__ __forceinline__ void init() {
#pragma unroll
        for (int k = 0; k < NP; ++k) v[k] = 0;
        ovf = 0;
    }
    __device__ __forceinline__ void add(int pat, u128 c, bool o) {
#pragma unroll
        for (int k = 0; k < NP; ++k)
            if (k == pat) {
                bool oo = o;
                v[k] = add_ovf(v[k], c, oo);
                if (oo) ovf |= 1u << k;
            }
    }
};

// Result sink of a pass.  Reduction is contention-free: lanes -> warp
// (shuffles) -> block (shared memory) -> one BlockPartial per block; the last
// block to finish (ticket) sums the partials and writes the pass result.
struct BlockPartial {
    unsigned long long lo[FSGC_MAXPATS], hi[FSGC_MAXPATS];
    unsigned long long matches;
    unsigned int ovf, pad;
};

struct Sink {
    AccDev* acc;                    // [FSGC_MAXPATS] final result
    unsigned long long* matches;    // final core-match count
    BlockPartial* parts;            // [gridDim.x]
    unsigned int* ticket;
    int mode;                       // 0: partials + last block sums; 1: one atomic per block
};

template <int NP>
__device__ __noinline__ void block_publish(const AccN<NP> A, unsigned long long nmatch, const Sink S) {
    __shared__ unsigned long long s_lo[32][NP], s_hi[32][NP];
    __shared__ unsigned int s_ovf[32];
    __shared__ unsigned long long s_m[32];
    __shared__ int s_last;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    uint32_t om = A.ovf;
#pragma unroll
    for (int pi = 0; pi < NP; ++pi) {
        u128 v = A.v[pi];
        bool o = false;
        warp_reduce_u128(v, o);
        if (o) om |= 1u << pi;
        if (lane == 0) { s_lo[wid][pi] = u128_lo(v); s_hi[wid][pi] = u128_hi(v); }
    }
    om = __reduce_or_sync(FULLMASK, om);
#pragma unroll
    for (int o = 16; o; o >>= 1) nmatch += __shfl_down_sync(FULLMASK, nmatch, o);
    if (lane == 0) { s_ovf[wid] = om; s_m[wid] = nmatch; }
    __syncthreads();
    if (wid == 0) {
        BlockPartial* bp = S.parts + blockIdx.x;
        uint32_t bo = lane < nw ? s_ovf[lane] : 0u;
#pragma unroll
        for (int pi = 0; pi < NP; ++pi) {
            u128 v = lane < nw ? u128_make(s_lo[lane][pi], s_hi[lane][pi]) : (u128)0;
            bool o = false;
            warp_reduce_u128(v, o);
            if (o) bo |= 1u << pi;
            if (lane == 0) { bp->lo[pi] = u128_lo(v); bp->hi[pi] = u128_hi(v); }
        }
        bo = __reduce_or_sync(FULLMASK, bo);
        unsigned long long bm = lane < nw ? s_m[lane] : 0ull;
#pragma unroll
        for (int o = 16; o; o >>= 1) bm += __shfl_down_sync(FULLMASK, bm, o);
        if (S.mode == 1) {               // block totals straight into the result
            if (lane < NP) {
                const u128 v = u128_make(bp->lo[lane], bp->hi[lane]);
                if (v != 0 || ((bo >> lane) & 1)) atomic_add_u128(S.acc + lane, v, (bo >> lane) & 1);
            }
            if (lane == 0 && bm) atomicAdd(S.matches, bm);
            return;                      // uniform per block: s_last never set
        }
        if (lane == 0) {
            bp->ovf = bo;
            bp->matches = bm;
            __threadfence();
            const unsigned t = atomicAdd(S.ticket, 1u);
            s_last = (t == gridDim.x - 1);
        }
    }
    if (S.mode == 1) return;
    __syncthreads();
    // last block: warp w sums pattern w (and warp 0 the flags / matches)
    if (s_last) {
        __threadfence();
        const int nb = gridDim.x;
        if (wid == 0) {
            uint32_t fo = 0;
            unsigned long long fm = 0;
#pragma unroll 4
            for (int b = lane; b < nb; b += 32) {
                fo |= __ldcg(&S.parts[b].ovf);
                fm += __ldcg(&S.parts[b].matches);
            }
            fo = __reduce_or_sync(FULLMASK, fo);
#pragma unroll
            for (int o = 16; o; o >>= 1) fm += __shfl_down_sync(FULLMASK, fm, o);
            if (lane == 0) {
                *S.matches = fm;
                for (int pi = 0; pi < NP; ++pi) S.acc[pi].pad = fo;  // flags, folded below
            }
        }
        __syncthreads();
        for (int pi = wid; pi < NP; pi += nw) {
            u128 v = 0;
            bool o = false;
#pragma unroll 4
            for (int b = lane; b < nb; b += 32)
                v = add_ovf(v, u128_make(__ldcg(&S.parts[b].lo[pi]), __ldcg(&S.parts[b].hi[pi])), o);
            warp_reduce_u128(v, o);
            if (lane == 0) {
                const uint32_t fo = S.acc[pi].pad;
                S.acc[pi].lo = u128_lo(v);
                S.acc[pi].hi = u128_hi(v);
                S.acc[pi].ovf = (o || ((fo >> pi) & 1)) ? 1u : 0u;
            }
        }
    }
}

// ------------------------------------------------------------------------
// 1-vertex cores (k-stars, the 1- and 2-vertex patterns): one thread per
// root vertex, Venn = {deg(v)} (Sec. 3 k-star formula generalised by fc).
template <int NP>
__global__ void __launch_bounds__(256) vertex_core_kernel(GraphDev G, const __grid_constant__ CoreProg P, WorkDesc W,
                                                          const Sink S) {
    AccN<NP> acc;
    acc.init();
    unsigned long long nmatch = 0;
    const int64_t total = W.end - W.begin;
    const int64_t nchunks = (total + W.chunk - 1) / W.chunk;
    const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
    // chunk c of this shard = global chunk c * nshards + shard
    for (int64_t c = tid / W.chunk; ; c += nthreads / W.chunk) {
        int64_t g = c * W.nshards + W.shard;
        if (g >= nchunks) break;
        int64_t t = g * W.chunk + tid % W.chunk;
        if (t >= total) continue;
        const int64_t v = W.begin + t;
        const uint32_t deg = (uint32_t)(G.offs[v + 1] - G.offs[v]);
        if (W.degfilter && (int)deg < P.mindeg[0]) continue;
        ++nmatch;
        uint32_t venn[2] = {0, deg};
        for (int pi = 0; pi < P.nprog; ++pi) {
            const FringeProg fp = P.prog[pi];
            bool o = false;
            u128 c2 = fc_dispatch<4>(venn, P.q, fp, o);
            acc.add(fp.pat, c2, o);
        }
    }
    block_publish<NP>(acc, nmatch, S);
}

// ------------------------------------------------------------------------
// 2-vertex (edge) cores, two streaming passes per count:
//
// (A) support_kernel: c(e) = |N(u) & N(v)| for every edge e = (u < v), by
//     listing each triangle u < v < w exactly once from its lowest edge:
//     w in N+(u) & N+(v), N+(x) = neighbours with a larger (degree-ordered)
//     id -- short lists, O(m^1.5) total.  The lane owning (u,v) adds its
//     triangles to c(uv); c(uw), c(vw) receive atomics (their oriented
//     indices come from the match positions).  One lane per root edge;
//     roots whose shorter out-list exceeds kHeavy are collected by ballot and
//     processed by the whole warp (Listing 7 style).
// (B) edge_fc_kernel: lane per root edge, Venn = {du-1-c, dv-1-c, c}
//     (e(x) excludes u and v; v in N(u); u, v not in N(u) & N(v)), fc by
//     Sec. 3.1's closed form for every program; coalesced reads only.
constexpr int kHeavy = 32;

struct OrientDev {
    const int64_t* __restrict__ split;
    const int64_t* __restrict__ oofs;
};

__device__ __forceinline__ int64_t oidx(const OrientDev& O, int u, int64_t p) {
    return __ldg(O.oofs + u) + (p - __ldg(O.split + u));
}

// sequential merge / gallop of A = adj[a0, a0+na) and B = adj[b0, b0+nb);
// every common element: atomics on the oriented edges (ua, A-pos), (ub, B-pos)
__device__ __forceinline__ int support_seq(const int32_t* __restrict__ adj, const OrientDev& O, int ua, int64_t a0,
                                           int na, int ub, int64_t b0, int nb, int* __restrict__ sup) {
    if (na == 0 || nb == 0) return 0;
    if (na > nb) {
        int t = ua; ua = ub; ub = t;
        int64_t t0 = a0; a0 = b0; b0 = t0;
        int tn = na; na = nb; nb = tn;
    }
    const int64_t baseA = __ldg(O.oofs + ua) - __ldg(O.split + ua) ;
    const int64_t baseB = __ldg(O.oofs + ub) - __ldg(O.split + ub);
    int c = 0;
    if (nb > 8 * na) {                       // gallop A's elements through B
        int j = 0;
        for (int i = 0; i < na && j < nb; ++i) {
            const int x = __ldg(adj + a0 + i);
            int step = 1, hi = j;
            while (hi < nb && __ldg(adj + b0 + hi) < x) { j = hi + 1; hi += step; step <<= 1; }
            if (hi > nb) hi = nb;
            int lo = j, h2 = hi;
            while (lo < h2) {
                int mid = (lo + h2) >> 1;
                if (__ldg(adj + b0 + mid) < x) lo = mid + 1; else h2 = mid;
            }
            j = lo;
            if (j < nb && __ldg(adj + b0 + j) == x) {
                ++c;
                atomicAdd(sup + baseA + a0 + i, 1);
                atomicAdd(sup + baseB + b0 + j, 1);
                ++j;
            }
        }
        return c;
    }
    int i = 0, j = 0;
    int x = __ldg(adj + a0), y = __ldg(adj + b0);
    for (;;) {
        if (x < y) { if (++i == na) break; x = __ldg(adj + a0 + i); }
        else if (x > y) { if (++j == nb) break; y = __ldg(adj + b0 + j); }
        else {
            ++c;
            atomicAdd(sup + baseA + a0 + i, 1);
            atomicAdd(sup + baseB + b0 + j, 1);
            if (++i == na || ++j == nb) break;
            x = __ldg(adj + a0 + i);
            y = __ldg(adj + b0 + j);
        }
    }
    return c;
}

// whole warp: lanes over the shorter list, binary search in the longer
__device__ __forceinline__ int support_warp(const int32_t* __restrict__ adj, const OrientDev& O, int ua, int64_t a0,
                                            int na, int ub, int64_t b0, int nb, int* __restrict__ sup, int lane) {
    if (na > nb) {
        int t = ua; ua = ub; ub = t;
        int64_t t0 = a0; a0 = b0; b0 = t0;
        int tn = na; na = nb; nb = tn;
    }
    const int64_t baseA = __ldg(O.oofs + ua) - __ldg(O.split + ua);
    const int64_t baseB = __ldg(O.oofs + ub) - __ldg(O.split + ub);
    int c = 0;
    for (int s0 = 0; s0 < na; s0 += 32) {
        const int i = s0 + lane;
        bool hit = false;
        if (i < na) {
            const int x = __ldg(adj + a0 + i);
            int lo = 0, hi = nb;
            while (lo < hi) {
                int mid = (lo + hi) >> 1;
                if (__ldg(adj + b0 + mid) < x) lo = mid + 1; else hi = mid;
            }
            if (lo < nb && __ldg(adj + b0 + lo) == x) {
                hit = true;
                atomicAdd(sup + baseA + a0 + i, 1);
                atomicAdd(sup + baseB + b0 + lo, 1);
            }
        }
        c += __popc(__ballot_sync(FULLMASK, hit));
    }
    return c;
}

// Roots are taken in the graph's support order (oriented edges sorted by
// merge length out(u) + out(v), fsgc_graph.sorder): warp w takes the 32-root
// chunks w, w + NW, ..., so the lanes of a warp run merges of similar length
// (little divergence) and the heaviest chunks, at the end, spread over warps.
__global__ void __launch_bounds__(256) support_kernel(GraphDev G, OrientDev O, int64_t m, int* __restrict__ sup,
                                                      const int32_t* __restrict__ sorder,
                                                      const int32_t* __restrict__ ssrc,
                                                      const int32_t* __restrict__ sdst, int shard,
                                                      int nshards, unsigned long long* trace) {
    const int lane = threadIdx.x & 31;
    const unsigned long long t_start = trace ? gtimer() : 0;
    int nch = 0;
    const int64_t NW = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    // shard s of n takes the 32-root chunks s, s + n, ... (interleaved over
    // the merge-length order, so every shard gets the same cost mix)
    const int64_t nchunks = ((m + 31) >> 5) - shard;
    const int64_t mychunks = nchunks > 0 ? (nchunks + nshards - 1) / nshards : 0;
    for (int64_t vch = warp; vch < mychunks; vch += NW) {
        ++nch;
        const int64_t ch = vch * nshards + shard;
        const int64_t t = ch * 32 + lane;
        const bool valid = t < m;
        int64_t e = 0;
        int u = 0, v = 0, nu = 0, nv = 0;
        int64_t su = 0, sv = 0;
        if (valid) {
            e = __ldg(sorder + t);
            u = __ldg(ssrc + t);
            v = __ldg(sdst + t);
            su = __ldg(O.split + u); nu = (int)(__ldg(G.offs + u + 1) - su);
            sv = __ldg(O.split + v); nv = (int)(__ldg(G.offs + v + 1) - sv);
        }
        const bool heavy = valid && min(nu, nv) > kHeavy;
        int c = 0;
        if (valid && !heavy) c = support_seq(G.adj, O, u, su, nu, v, sv, nv, sup);
        unsigned hb = __ballot_sync(FULLMASK, heavy);
        while (hb) {
            const int who = __ffs(hb) - 1;
            hb &= hb - 1;
            const int wu = __shfl_sync(FULLMASK, u, who), wv = __shfl_sync(FULLMASK, v, who);
            const int64_t wsu = __shfl_sync(FULLMASK, su, who), wsv = __shfl_sync(FULLMASK, sv, who);
            const int wnu = __shfl_sync(FULLMASK, nu, who), wnv = __shfl_sync(FULLMASK, nv, who);
            const int cc = support_warp(G.adj, O, wu, wsu, wnu, wv, wsv, wnv, sup, lane);
            if (lane == who) c = cc;
        }
        if (valid && c) atomicAdd(sup + e, c);
    }
    if (trace && lane == 0) {
        unsigned smid;
        asm volatile("mov.u32 %0, %smid;" : "=r"(smid));
        unsigned long long* tr = trace + 8 * warp;
        tr[0] = t_start; tr[1] = gtimer(); tr[2] = smid; tr[3] = (unsigned long long)nch;
    }
}

// One program of the Sec. 3.1 closed form, out of line: the kernels are short
// and latency-bound, so a compact hot path (instruction-cache footprint)
// matters more than call overhead.  `small`: the 64-bit bound holds.
__device__ __noinline__ u128 edge_prog_eval(uint64_t nu, uint64_t nv, uint64_t nuv, uint32_t w, bool small,
                                            bool& o) {
    const int k = w & 255, l = (w >> 8) & 255, m = (w >> 16) & 255;
    if (small) return (u128)edge_formula<Exact64>(nu, nv, nuv, k, l, m, o);
    return edge_formula<Checked128>(nu, nv, nuv, k, l, m, o);
}

// oriented index of the directed CSR entry `item` = (u, v)
__device__ __forceinline__ int64_t edge_of_entry(const GraphDev& G, const OrientDev& O, int u, int v, int64_t item) {
    if (u < v) return oidx(O, u, item);
    int64_t lo = __ldg(O.split + v), hi = __ldg(G.offs + v + 1);   // position of u in N+(v)
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (__ldg(G.adj + mid) < u) lo = mid + 1; else hi = mid;
    }
    return oidx(O, v, lo);
}

constexpr int kEdgeILP = 4;   // root edges per lane per iteration (independent loads in flight)

// Sec. 3.1's closed form over binomial rows.  With the multinomial identity
//   C(n,i) C(n-i,j) C(n-i-j,m) = C(n, i+j+m) (i+j+m)! / (i! j! m!)
// the last displayed formula of Sec. 3.1 becomes
//   fc(k,l,m) = sum_{i<=k, j<=l} C(nu,k-i) C(nv,l-j) C(nuv,i+j+m) (i+j+m)!/(i! j! m!),
// a sum of products of three row entries Ra[a] = C(nu,a), Rb[b] = C(nv,b),
// Rc[c] = C(nuv,c).  The host lists every (pattern, a, b, c, coefficient)
// term of every program of the pass once (terms of one pattern merged), so a
// root costs three short rows plus one multiply-add chain per term, shared by
// all patterns and programs of the pass.
constexpr int kMaxEdgeTerms = 160;
constexpr int kMaxRowEntries = 24;   // (ka+1) + (kb+1) + (kc+1)
struct EdgeTerm {
    uint8_t a, b, c, pat;
    uint32_t pad;
    uint64_t coef;
};
struct EdgeTerms {
    int32_t n;              // terms; 0: table path off (checked per-program path)
    int32_t ka, kb, kc;     // row lengths - 1
    int32_t kmax;           // max fringes of one program (64-bit bound, fc.cuh)
    int32_t pad;
    EdgeTerm t[kMaxEdgeTerms];
};

// exact division by t <= 63 of a multiple of t: shift out the 2-adic part,
// multiply by the inverse of the odd part mod 2^64 (filled by ensure_binom_table)
__constant__ uint64_t c_inv_odd[64];     // mod 2^64
__constant__ uint64_t c_inv_odd_hi[64];  // high words of the inverses mod 2^128
__constant__ uint32_t c_tz[64];

__device__ __forceinline__ uint64_t inv_odd(int t, uint64_t) { return c_inv_odd[t]; }
__device__ __forceinline__ u128 inv_odd(int t, u128) { return u128_make(c_inv_odd[t], c_inv_odd_hi[t]); }

// R[t * stride] = C(n, t), t = 0..K, in arithmetic mod 2^bits(W); exact when
// n^K < 2^(bits - 1) (caller's bound): every r * (n - t + 1) <= n^t then fits
template <class W>
__device__ __forceinline__ void binom_row(uint64_t n, int K, W* R, int stride) {
    W r = 1;
    R[0] = 1;
    for (int t = 1; t <= K; ++t) {
        r = ((r * (W)(n - (uint64_t)t + 1)) >> c_tz[t]) * inv_odd(t, r);
        R[t * stride] = r;
    }
}

// every term of the pass on one root's rows, arithmetic mod 2^bits(W): exact
// because every program's fc is below N^K < 2^(bits - 1) (caller's bound) and
// a pattern has at most |Aut(edge)| = 2 programs, so each pattern's sum fits
template <class W, int NP>
__device__ __forceinline__ void edge_terms_eval(uint64_t nu, uint64_t nv, uint64_t nuv, const EdgeTerms& T, W* R,
                                                int stride, AccN<NP>& acc) {
    W* Ra = R;
    W* Rb = Ra + (T.ka + 1) * stride;
    W* Rc = Rb + (T.kb + 1) * stride;
    binom_row<W>(nu, T.ka, Ra, stride);
    binom_row<W>(nv, T.kb, Rb, stride);
    binom_row<W>(nuv, T.kc, Rc, stride);
    W sum = 0;
    int cur = T.t[0].pat;
    for (int t = 0; t < T.n; ++t) {
        const EdgeTerm e = T.t[t];
        if (e.pat != cur) { acc.add(cur, (u128)sum, false); sum = 0; cur = e.pat; }
        sum += (W)e.coef * Ra[e.a * stride] * Rb[e.b * stride] * Rc[e.c * stride];
    }
    acc.add(cur, (u128)sum, false);
}

template <int NP>
__global__ void __launch_bounds__(256) edge_fc_kernel(GraphDev G, OrientDev O, const __grid_constant__ CoreProg P, WorkDesc W,
                                                      const int* __restrict__ sup, const __grid_constant__ EdgeTerms T,
                                                      const Sink S) {
    extern __shared__ u128 s_rows[];                 // [row entry][thread] (table path)
    // program table (checked fallback path): k | l << 8 | m << 16 | pattern << 24
    __shared__ uint32_t s_prog[FSGC_MAXPROG];
    __shared__ uint32_t s_q[8][64][3];               // per warp: queued roots (nu, nv, nuv)
    __shared__ int s_minm;
    if (threadIdx.x == 0) {
        int minm = 255;
        for (int pi = 0; pi < P.nprog; ++pi) minm = min(minm, (int)P.em[pi]);
        s_minm = minm;
    }
    if (threadIdx.x < P.nprog)
        s_prog[threadIdx.x] = P.ek[threadIdx.x] | (P.el[threadIdx.x] << 8) | (P.em[threadIdx.x] << 16) |
                              ((uint32_t)P.prog[threadIdx.x].pat << 24);
    __syncthreads();
    const int nprog = P.nprog;
    const int minm = s_minm;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int stride = blockDim.x;
    AccN<NP> acc;
    acc.init();
    unsigned long long nmatch = 0;
    int cnt = 0;                                      // queue length (warp-uniform)

    // lanes < take each evaluate one queued root, then the rest moves up
    auto drain = [&](int take) {
        __syncwarp();
        if (lane < take) {
            const uint64_t nu = s_q[wib][lane][0], nv = s_q[wib][lane][1], nuv = s_q[wib][lane][2];
            const int nbits = T.n > 0 ? bitlen64(nu + nv + nuv) * T.kmax : 1 << 20;
            if (nbits <= 63) {
                // same byte layout as the u128 rows (threads of another tier share the
                // buffer): entry t of this thread in the low half of its u128 slot
                edge_terms_eval<uint64_t>(nu, nv, nuv, T, (uint64_t*)(s_rows + threadIdx.x), 2 * stride, acc);
            } else if (nbits <= 127) {
                edge_terms_eval<u128>(nu, nv, nuv, T, (u128*)s_rows + threadIdx.x, stride, acc);
            } else {
                for (int pi = 0; pi < nprog; ++pi) {
                    const uint32_t w = s_prog[pi];
                    bool o = false;
                    const u128 f = edge_prog_eval(nu, nv, nuv, w, false, o);
                    acc.add((int)(w >> 24), f, o);
                }
            }
        }
        __syncwarp();
        const int rest = cnt - take;
        if (lane < rest) {
#pragma unroll
            for (int x = 0; x < 3; ++x) s_q[wib][lane][x] = s_q[wib][take + lane][x];
        }
        cnt = rest;
        __syncwarp();
    };

    const int64_t total = W.end - W.begin;
    // this shard owns the 32-item chunks g = c * nshards + shard; its items are
    // numbered L = c * 32 + lane and walked grid-stride, kEdgeILP at a time,
    // transposed (lane l of warp w takes local item l * NW + w of each slice)
    // so the hub roots (clustered at the end of the degree order) spread out
    const int64_t nchunks = (total + 31) / 32;
    const int64_t mychunks = nchunks > W.shard ? (nchunks - W.shard + W.nshards - 1) / W.nshards : 0;
    const int64_t nloc = mychunks * 32;
    const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const bool oriented = P.root_mode == ROOT_ORIENTED;
    const int64_t NW = nthreads >> 5;
    const int64_t tpos = (int64_t)lane * NW + warp;
    for (int64_t L0 = 0; L0 < nloc; L0 += nthreads * kEdgeILP) {
        int u[kEdgeILP], v[kEdgeILP], c[kEdgeILP];
        int64_t itm[kEdgeILP];
        bool ok[kEdgeILP];
#pragma unroll
        for (int j = 0; j < kEdgeILP; ++j) {           // 1: root edges (+ support, coalesced)
            const int64_t L = L0 + j * nthreads + tpos;
            const int64_t t = ((L >> 5) * W.nshards + W.shard) * 32 + (L & 31);
            ok[j] = L < nloc && t < total;
            itm[j] = W.begin + (ok[j] ? t : 0);
            if (oriented) {
                u[j] = __ldg(G.osrc + itm[j]); v[j] = __ldg(G.odst + itm[j]);
                c[j] = __ldg(sup + itm[j]);
            } else {
                u[j] = __ldg(G.row + itm[j]); v[j] = __ldg(G.adj + itm[j]);
            }
        }
        if (!oriented) {
#pragma unroll
            for (int j = 0; j < kEdgeILP; ++j) c[j] = __ldg(sup + edge_of_entry(G, O, u[j], v[j], itm[j]));
        }
        int du[kEdgeILP], dv[kEdgeILP];
#pragma unroll
        for (int j = 0; j < kEdgeILP; ++j) {           // 2: degrees, only where a program can match
            du[j] = dv[j] = 0;
            if (ok[j] && (c[j] >= minm || !W.degfilter)) {
                du[j] = (int)(__ldg(G.offs + u[j] + 1) - __ldg(G.offs + u[j]));
                dv[j] = (int)(__ldg(G.offs + v[j] + 1) - __ldg(G.offs + v[j]));
            }
        }
#pragma unroll
        for (int j = 0; j < kEdgeILP; ++j) {           // 3: Venn diagrams -> warp queue
            bool work = false;
            if (ok[j]) {
                const bool pass = !W.degfilter || (c[j] >= minm && du[j] >= P.mindeg[0] && dv[j] >= P.mindeg[1]);
                if (pass) ++nmatch;
                work = pass && c[j] >= minm;           // every program needs >= minm wedge fringes
            }
            const unsigned wm = __ballot_sync(FULLMASK, work);
            if (work) {
                const int slot = cnt + __popc(wm & ((1u << lane) - 1));
                s_q[wib][slot][0] = (uint32_t)(du[j] - 1 - c[j]);
                s_q[wib][slot][1] = (uint32_t)(dv[j] - 1 - c[j]);
                s_q[wib][slot][2] = (uint32_t)c[j];
            }
            cnt += __popc(wm);
            if (cnt >= 32) drain(32);
        }
    }
    if (cnt) drain(cnt);
    block_publish<NP>(acc, nmatch, S);
}

// ------------------------------------------------------------------------
// Venn term tables (triangle and general cores).  Listing 5 distributes the
// k_t fringes of every type over the Venn regions r covering its anchor set;
// with x_{t,r} fringes of type t in region r and s_r = sum_t x_{t,r},
//   fc = sum_x prod_r C(n_r; x_{1,r}, .., x_{T,r}, n_r - s_r)
//      = sum_s M(s) prod_r C(n_r, s_r),   M(s) = sum_{x -> s} prod_r s_r! / prod_t x_{t,r}!
// (the multinomial split of each region).  M depends on the pattern only, so
// the host enumerates Listing 5's tree ONCE per pass, merging the terms of
// every program (coset of Aut_C') of a pattern; a core match then costs its
// binomial rows C(n_r, 0..max s_r) plus one product chain per distinct s --
// e.g. Fig. 4 on the triangle core: 2,889 terms instead of 6 x 18,000
// Listing 5 leaves.
constexpr int kMaxVennTerms = 8192;
constexpr int kMaxVennRows = 64;
constexpr int kMaxVennNz = 14;
struct VTerm {
    uint64_t coef;
    uint8_t pat, nz;
    uint8_t off[kMaxVennNz];     // row entries (base[r] + s_r - 1) of the regions with s_r > 0
};
// Z-term table (triangle cores whose every program is a single fringe type
// or has all k = 1): fc from the intersection sizes Z[A] = |cap_{x in A} e(x)|
// of the core-position sets A -- for a triangle core Z[{x}] = deg(x) - 2,
// Z[{x,y}] = c(xy) - 1, Z[{u,v,w}] = t -- instead of the Venn diagram:
//   single type (A, k):   fc = C(Z[A], k)
//   all k = 1:            fc = sum_pi coef(pi) prod_B Z[A_B]  (partition
//                         lattice, Moebius inversion -- PartTerm)
// A term: signed coefficient x product of row entries C(Z[cm], j); terms of
// the same pattern and the same factors are merged across programs.
constexpr int kMaxZTerms = 512;
struct ZTerm {
    int64_t coef;
    uint8_t pat, nf;
    uint8_t f[6];                // factors C(Z[cm], j), coded cm << 5 | j (j <= 31)
};

struct VennDev {
    const VTerm* __restrict__ terms;
    int32_t n;                   // terms; 0: table off (per-program Listing 5)
    int32_t nrows;               // row entries per core match (C(n_r, j), j >= 1)
    float slack;                 // log2(programs per pattern) + margin
    int32_t warp;                // 1: one diagram per warp (large tables), 0: one per lane
    uint8_t maxs[64];            // per region: max s_r (0: no row)
    uint8_t base[64];            // per region: first row entry
    // Z-term table (triangle cores; zn == 0: off)
    const ZTerm* __restrict__ zterms;
    int32_t zn;
    int32_t znrows;
    int32_t zneed7;              // some factor uses Z[{u,v,w}] = t
    int32_t zk;                  // max fringes of one program (bound)
    uint8_t zmaxj[8];            // per core mask cm: max j of C(Z[cm], j)
    uint8_t zbase[8];            // per core mask cm: first row entry (unused by the row-free evaluation)
    uint16_t zoff[FSGC_MAXPATS + 1];   // terms of pattern p: [zoff[p], zoff[p+1]) (sorted by pattern)
    int32_t zmax64, zmax128;     // largest max-degree of a leaf whose tier bound
                                 // zk log2(Z + 1) + slack stays below 55 / 119
    int32_t zmax64p[FSGC_MAXPATS];   // per pattern: largest leaf max-degree whose
                                     // pattern sum and binomials fit 64 bits
};

// log2 upper bound of one pattern's fc sum on this diagram:
// max over programs of sum_t k_t log2(Z[A_t] + 1), Z[A] = vertices covering A
// (prod_t C(Z_t, k_t) bounds each program's fc); the caller adds T.slack
__device__ __noinline__ float venn_bound_log2(const uint32_t* venn, int q, const CoreProg& P) {
    const int V = 1 << q;
    uint32_t Z[64];
    for (int A = 0; A < V; ++A) Z[A] = A ? venn[A] : 0;
    for (int bb = 0; bb < q; ++bb)
        for (int A = 0; A < V; ++A)
            if (!(A >> bb & 1)) Z[A] += Z[A | (1 << bb)];
    float mx = 0.f;
    for (int pi = 0; pi < P.nprog; ++pi) {
        const FringeProg& fp = P.prog[pi];
        float b = 0.f;
        for (int t = 0; t < fp.s; ++t) b += (float)fp.k[t] * log2f((float)Z[fp.anch[t]] + 1.f);
        mx = fmaxf(mx, b);
    }
    return mx;
}

// one diagram, every term of the pass, arithmetic mod 2^bits(W): exact when
// each pattern's fc sum (>= every term, every partial sum) is below
// 2^(bits - 9): then every used row entry C(n, s) and s * C(n, s) fit too
template <class W, class ACC>
__device__ __forceinline__ void venn_terms_eval(const uint32_t* venn, int V, const VennDev& T, W* R, int stride,
                                                ACC& acc) {
    for (int r = 1; r < V; ++r) {      // R[base[r] + j - 1] = C(n_r, j), j = 1..maxs[r]
        const int K = T.maxs[r];
        if (!K) continue;
        const uint64_t n = venn[r];
        W* Rr = R + T.base[r] * stride;
        W c = 1;
        for (int j = 1; j <= K; ++j) {
            c = ((c * (W)(n - (uint64_t)j + 1)) >> c_tz[j]) * inv_odd(j, c);
            Rr[(j - 1) * stride] = c;
        }
    }
    W sum = 0;
    int cur = T.terms[0].pat;
    for (int t = 0; t < T.n; ++t) {
        const VTerm* e = T.terms + t;
        const uint64_t cf = __ldg(&e->coef);
        const uint2 hd = __ldg(reinterpret_cast<const uint2*>(e) + 1);
        const uint2 tl = __ldg(reinterpret_cast<const uint2*>(e) + 2);
        const int pat = hd.x & 255, nz = (hd.x >> 8) & 255;
        if (pat != cur) { acc.add(cur, (u128)sum, false); sum = 0; cur = pat; }
        // off[0..1] in hd.x bits 16..31, off[2..5] in hd.y, off[6..13] in tl
        W pr = (W)cf;
        const uint32_t words[4] = {hd.x >> 16, hd.y, tl.x, tl.y};
#pragma unroll
        for (int i = 0; i < kMaxVennNz; ++i) {   // constant shifts, no local memory
            if (i >= nz) break;
            const int o = i < 2 ? (int)((words[0] >> (8 * i)) & 255)
                                : (int)((words[1 + (i - 2) / 4] >> (8 * ((i - 2) & 3))) & 255);
            pr *= R[o * stride];
        }
        sum += pr;
    }
    acc.add(cur, (u128)sum, false);
}

// The same table, one diagram per WARP: the lanes owning a region build its
// binomial row in the warp's shared buffer, then take the terms strided (each
// lane's subsequence stays grouped by pattern, and its partial sums are
// bounded by the pattern's sum, so the tier argument above holds per lane).
template <class W, class ACC>
__device__ __forceinline__ void venn_warp_terms(const uint32_t* venn, int V, const VennDev& T, W* R, int lane,
                                                ACC& acc) {
    for (int r = 1 + lane; r < V; r += 32) {
        const int K = T.maxs[r];
        if (!K) continue;
        const uint64_t n = venn[r];
        W* Rr = R + T.base[r];
        W c = 1;
        for (int j = 1; j <= K; ++j) {
            c = ((c * (W)(n - (uint64_t)j + 1)) >> c_tz[j]) * inv_odd(j, c);
            Rr[j - 1] = c;
        }
    }
    __syncwarp();
    W sum = 0;
    int cur = -1;
    for (int t = lane; t < T.n; t += 32) {
        const VTerm* e = T.terms + t;
        const uint64_t cf = __ldg(&e->coef);
        const uint2 hd = __ldg(reinterpret_cast<const uint2*>(e) + 1);
        const uint2 tl = __ldg(reinterpret_cast<const uint2*>(e) + 2);
        const int pat = hd.x & 255, nz = (hd.x >> 8) & 255;
        if (pat != cur) {
            if (cur >= 0) acc.add(cur, (u128)sum, false);
            sum = 0;
            cur = pat;
        }
        W pr = (W)cf;
        const uint32_t words[4] = {hd.x >> 16, hd.y, tl.x, tl.y};
#pragma unroll
        for (int i = 0; i < kMaxVennNz; ++i) {
            if (i >= nz) break;
            const int o = i < 2 ? (int)((words[0] >> (8 * i)) & 255)
                                : (int)((words[1 + (i - 2) / 4] >> (8 * ((i - 2) & 3))) & 255);
            pr *= R[o];
        }
        sum += pr;
    }
    if (cur >= 0) acc.add(cur, (u128)sum, false);
    __syncwarp();
}

// venn_bound_log2 with the programs split over the lanes (warp max)
__device__ __forceinline__ float venn_bound_log2_warp(const uint32_t* venn, int q, const CoreProg& P, int lane) {
    const int V = 1 << q;
    float lz[64];
    {
        uint32_t Z[64];
        for (int A = 0; A < V; ++A) Z[A] = A ? venn[A] : 0;
        for (int bb = 0; bb < q; ++bb)
            for (int A = 0; A < V; ++A)
                if (!(A >> bb & 1)) Z[A] += Z[A | (1 << bb)];
        for (int A = 0; A < V; ++A) lz[A] = log2f((float)Z[A] + 1.f);
    }
    float mx = 0.f;
    for (int pi = lane; pi < P.nprog; pi += 32) {
        const FringeProg& fp = P.prog[pi];
        float b = 0.f;
        for (int t = 0; t < fp.s; ++t) b += (float)fp.k[t] * lz[fp.anch[t]];
        mx = fmaxf(mx, b);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(FULLMASK, mx, o));
    return mx;
}

// fc of one diagram by the whole warp: table tiers, else checked Listing 5
// with the programs split over the lanes
template <int STACK, class ACC>
__device__ __forceinline__ void venn_fc_warp(uint32_t* vloc, int q, const CoreProg& P, const VennDev& VD,
                                             u128* rows, int lane, ACC& acc) {
    const int V = 1 << q;
    const float bnd = venn_bound_log2_warp(vloc, q, P, lane) + VD.slack;
    if (bnd < 55.f) {
        venn_warp_terms<uint64_t>(vloc, V, VD, reinterpret_cast<uint64_t*>(rows), lane, acc);
    } else if (bnd < 119.f) {
        venn_warp_terms<u128>(vloc, V, VD, rows, lane, acc);
    } else {
        for (int pi = lane; pi < P.nprog; pi += 32) {
            const FringeProg fp = P.prog[pi];
            bool o = false;
            const u128 f = fc_dispatch<STACK>(vloc, q, fp, o);
            acc.add(fp.pat, f, o);
        }
    }
}

// ------------------------------------------------------------------------
// Triangle cores (p = 3, all pairs adjacent; symmetry broken u < v < w).
//
// Enumeration: one lane per oriented root edge (u, v), merging the short
// degree-oriented out-lists N+(u), N+(v): each common w is a triangle found
// exactly once (from its lowest edge).  Lanes advance to their next match,
// the warp ballots the lanes that found one (Listing 7) and appends those
// core matches to a per-warp leaf buffer in shared memory.
// Venn (Sec. 3.3): with c(xy) = |N(x) & N(y)| from the support pass and
// t = |N(u) & N(v) & N(w)| (one triple intersection, scanning the smallest
// list N(u) -- u has the lowest degree -- against v, w via hub bitmaps or
// galloping cursors), the 7 regions of e(u), e(v), e(w) (core vertices
// excluded; every core vertex is adjacent to the other two) are
//   uvw = t, uv = c(uv)-1-t, uw = c(uw)-1-t, vw = c(vw)-1-t,
//   u = deg(u)-2-uv-uw-t (and likewise v, w).
// fc: Listing 5 over (leaf, program) pairs spread across the lanes.
struct HubDev {
    int64_t base, words;
    const uint32_t* __restrict__ bits;
};

// galloping membership cursor over a sorted adjacency list (queries ascending)
struct Cursor {
    const int32_t* __restrict__ L;
    const uint32_t* __restrict__ bm;   // hub bitmap row or nullptr
    int len, j;
    __device__ __forceinline__ void init(const GraphDev& G, const HubDev& H, int y) {
        if (y >= H.base) {
            bm = H.bits + (int64_t)(y - H.base) * H.words;
            L = nullptr; len = 0; j = 0;
        } else {
            bm = nullptr;
            const int64_t b = __ldg(G.offs + y);
            L = G.adj + b;
            len = (int)(__ldg(G.offs + y + 1) - b);
            j = 0;
        }
    }
    __device__ __forceinline__ bool has(int x) {
        if (bm) return (__ldg(bm + (x >> 5)) >> (x & 31)) & 1u;
        int lo = j;
        if (lo >= len) return false;
        int y = __ldg(L + lo);
        if (y >= x) { j = lo; return y == x; }
        int step = 1, hi = lo + 1;
        while (hi < len && __ldg(L + hi) < x) { lo = hi; step <<= 1; hi = lo + step; }
        if (hi > len) hi = len;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (__ldg(L + mid) < x) lo = mid; else hi = mid;
        }
        j = hi;
        return hi < len && __ldg(L + hi) == x;
    }
};

__device__ __forceinline__ bool member(const GraphDev& G, const HubDev& H, int y, int x) {
    if (y >= H.base) return (__ldg(H.bits + (int64_t)(y - H.base) * H.words + (x >> 5)) >> (x & 31)) & 1u;
    const int64_t b = __ldg(G.offs + y);
    return contains(G.adj + b, (int)(__ldg(G.offs + y + 1) - b), x);
}

constexpr int kTriWarps = 8;   // warps per block of the triangle-core kernels
constexpr int kTriLight = 32;     // N(u) longer than this: warp-cooperative triple intersection
constexpr int kTriStack = 32;

#include "listing.cuh"

// ------------------------------------------------------------------------
// General cores (p >= 3): one warp per root edge (atomic chunk queue, heavy
// roots first), depth-first core matching with the Listing 7 ballot scheme.
// Core matches are buffered per warp (32 leaves) and their Venn diagrams
// computed ONE LANE PER LEAF (warp-cooperatively only for long lists):
//   * anchors sorted by degree at run time; the lists of all but the two
//     largest-degree anchors are scanned, each element tested against the
//     later anchors (galloping cursors / hub bitmaps) -> raw histogram H
//     (Sec. 3.6: only later anchors are searched, then corrected);
//   * the last two anchors' pair count is the per-edge support when they are
//     a core edge (else one more scan), singletons are degrees;
//   * raw regions (core vertices included) follow by the Sec. 3.6 correction
//     and inclusion-exclusion; each core vertex is then removed from the
//     region of anchors it is adjacent to (e(x) excludes the core).
// fc per (leaf, program) pair across the lanes: the partition-lattice terms
// when every fringe type has k = 1, else Listing 5.
struct TermDev {
    const PartTerm* __restrict__ terms;
    const int32_t* __restrict__ off;     // per program
    const int32_t* __restrict__ cnt;     // per program, < 0: Listing 5
};

constexpr int kCoreWarps = 4;
constexpr int kCoreLight = 48;   // scan work above this per leaf: warp-cooperative

// oriented index of the graph edge {a, b} (must exist)
__device__ __forceinline__ int64_t edge_index(const GraphDev& G, const OrientDev& O, int a, int b) {
    const int lo = min(a, b), hi = max(a, b);
    int64_t l = __ldg(O.split + lo), h = __ldg(G.offs + lo + 1);
    while (l < h) {
        const int64_t mid = (l + h) >> 1;
        if (__ldg(G.adj + mid) < hi) l = mid + 1; else h = mid;
    }
    return __ldg(O.oofs + lo) + (l - __ldg(O.split + lo));
}

// partition-lattice fc: Z[A] = sum_{e >= A} venn[e]; fc = sum coef prod Z[mask].
// Exact when every product and partial sum stays below 2^126 in magnitude,
// which the rising-factorial bound (N + s)^s <= 2^126 guarantees (N = Z[0]);
// returns false when the bound does not hold -- the caller then evaluates the
// program by checked Listing 5 instead (exact or flagged, never a
// conservative overflow)
__device__ __noinline__ bool fc_partition(const uint32_t* venn, int q, const PartTerm* __restrict__ T, int nt,
                                          u128& out) {
    int64_t Z[64];
    const int V = 1 << q;
    for (int A = 0; A < V; ++A) Z[A] = A ? venn[A] : 0;
    for (int bb = 0; bb < q; ++bb)
        for (int A = 0; A < V; ++A)
            if (!(A >> bb & 1)) Z[A] += Z[A | (1 << bb)];
    uint64_t N = (uint64_t)Z[0];
    int smax = 0;
    for (int i = 0; i < nt; ++i) smax = max(smax, (int)T[i].nb);   // the finest partition: s blocks
    const int bits = bitlen64(N + (uint64_t)smax) * smax;
    if (bits <= 62) {
        int64_t tot = 0;
        for (int i = 0; i < nt; ++i) {
            int64_t pr = T[i].coef;
            for (int bb = 0; bb < T[i].nb; ++bb) pr *= Z[T[i].mask[bb]];
            tot += pr;
        }
        out = (u128)(uint64_t)tot;       // the count is non-negative
        return true;
    }
    if (bits > 126) return false;
    u128 tot = 0;                        // signed 128-bit (two's complement)
    for (int i = 0; i < nt; ++i) {
        const bool neg = T[i].coef < 0;
        u128 pr = (u128)(uint64_t)(neg ? -(int64_t)T[i].coef : T[i].coef);
        for (int bb = 0; bb < T[i].nb; ++bb) pr *= (u128)(uint64_t)Z[T[i].mask[bb]];
        tot = neg ? tot - pr : tot + pr;
    }
    out = tot;
    return true;
}

template <int NP>
__global__ void __launch_bounds__(kCoreWarps * 32) core_kernel(GraphDev G, OrientDev O, HubDev H,
                                                                const __grid_constant__ CoreProg P, WorkDesc W,
                                                                const int* __restrict__ sup, TermDev TD,
                                                                const __grid_constant__ VennDev VD, const Sink S,
                                                                unsigned long long* queue) {
    extern __shared__ uint32_t smem[];
    __shared__ u128 s_vrows[kCoreWarps][kMaxVennRows];   // Venn-table binomial rows, per warp
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int q = P.q, V = 1 << q, p = P.p, nprog = P.nprog;
    uint32_t* s_leaf = smem + wib * (32 * FSGC_MAXC);                       // [32][MAXC]
    uint32_t* s_venn = smem + kCoreWarps * 32 * FSGC_MAXC + wib * (32 * V);  // [32][V]
    AccN<NP> acc;
    acc.init();
    unsigned long long nmatch = 0;
    int cnt = 0;

    int emb[FSGC_MAXC];
    int64_t eoff[FSGC_MAXC];
    int edeg[FSGC_MAXC];
    int64_t cur[FSGC_MAXC], endp[FSGC_MAXC];
    uint32_t pend[FSGC_MAXC];
    int pivl[FSGC_MAXC];
    // core adjacency of positions (pattern core edges => graph edges)
    uint32_t cadj[FSGC_MAXC];
#pragma unroll
    for (int i = 0; i < FSGC_MAXC; ++i) cadj[i] = 0;
    for (int i = 1; i < p; ++i)
        for (int j = 0; j < i; ++j)
            if ((P.back[i] >> j) & 1) { cadj[i] |= 1u << j; cadj[j] |= 1u << i; }

    // ---- Venn of leaf li (one lane) -> s_venn
    auto venn_lane = [&](int li, bool heavy_path) {
        int a[FSGC_MAXQ], d[FSGC_MAXQ], pos[FSGC_MAXQ];
        for (int bb = 0; bb < q; ++bb) {
            pos[bb] = P.anchor_pos[bb];
            a[bb] = (int)s_leaf[li * FSGC_MAXC + pos[bb]];
            d[bb] = (int)(__ldg(G.offs + a[bb] + 1) - __ldg(G.offs + a[bb]));
        }
        int pi_[FSGC_MAXQ];                       // anchors by degree ascending
        for (int bb = 0; bb < q; ++bb) pi_[bb] = bb;
        for (int i = 1; i < q; ++i)
            for (int j = i; j > 0 && d[pi_[j]] < d[pi_[j - 1]]; --j) { int t = pi_[j]; pi_[j] = pi_[j - 1]; pi_[j - 1] = t; }
        int32_t R[64];
        for (int k = 0; k < V; ++k) R[k] = 0;
        const bool pair_adj = q >= 2 && ((cadj[pos[pi_[q - 2]]] >> pos[pi_[q - 1]]) & 1);
        const int nscan = q >= 2 ? (pair_adj ? q - 2 : q - 1) : 0;
        if (!heavy_path) {
            for (int i = 0; i < nscan; ++i) {      // H[(1<<i) | later-mask], permuted bits
                Cursor cs[FSGC_MAXQ];
                for (int j = i + 1; j < q; ++j) cs[j].init(G, H, a[pi_[j]]);
                const int64_t b0 = __ldg(G.offs + a[pi_[i]]);
                for (int k = 0; k < d[pi_[i]]; ++k) {
                    const int x = __ldg(G.adj + b0 + k);
                    int m = 1 << i;
                    for (int j = i + 1; j < q; ++j)
                        if (cs[j].has(x)) m |= 1 << j;
                    R[m] += 1;
                }
            }
        } else {
            for (int k = 0; k < V; ++k) R[k] = (int32_t)s_venn[li * V + k];   // H from the warp pass
        }
        // Sec. 3.6 correction: entries with lowest bit i < nscan are exact
        // once the entries with a lower lowest bit are
        for (int i = 0; i < nscan; ++i)
            for (int t = V - 1; t > 0; --t) {
                if ((__ffs(t) - 1) != i) continue;
                const int low = (1 << i) - 1;
                for (int E = low; E > 0; E = (E - 1) & low) R[t] -= R[E | t];
            }
        // the unscanned anchors: pair from the support, singletons from degrees
        if (q >= 2 && pair_adj) {
            const int i = q - 2, hb = (1 << (q - 2)) | (1 << (q - 1));
            int r = __ldg(sup + edge_index(G, O, a[pi_[q - 2]], a[pi_[q - 1]]));
            const int low = (1 << i) - 1;
            for (int E = low; E > 0; E = (E - 1) & low) r -= R[E | hb];
            R[hb] = r;
        }
        for (int i = nscan; i < q; ++i) {
            int r = d[pi_[i]];
            for (int t = V - 1; t > 0; --t)
                if (((t >> i) & 1) && t != (1 << i)) r -= R[t];
            R[1 << i] = r;
        }
        // remove the core vertices from their regions (e(x) excludes the core)
        for (int y = 0; y < p; ++y) {
            const int vy = (int)s_leaf[li * FSGC_MAXC + y];
            int m = 0;
            for (int i = 0; i < q; ++i) {
                const int py = pos[pi_[i]];
                if (py == y) continue;                        // no self loops
                const bool adj = ((cadj[y] >> py) & 1) || member(G, H, a[pi_[i]], vy);
                if (adj) m |= 1 << i;
            }
            if (m) R[m] -= 1;
        }
        // back to the programs' Venn bit order
        for (int t = 1; t < V; ++t) {
            int tb = 0;
            for (int i = 0; i < q; ++i)
                if ((t >> i) & 1) tb |= 1 << pi_[i];
            s_venn[li * V + tb] = (uint32_t)R[t];
        }
        s_venn[li * V] = 0;
    };

    auto flush = [&]() {
        __syncwarp();
        const int li = lane;
        bool mine = li < cnt, heavy = false;
        if (mine) {                              // scan work of this leaf
            int d2[FSGC_MAXQ], ds = 0;
            for (int bb = 0; bb < q; ++bb) {
                const int v = (int)s_leaf[li * FSGC_MAXC + P.anchor_pos[bb]];
                d2[bb] = (int)(__ldg(G.offs + v + 1) - __ldg(G.offs + v));
            }
            for (int i = 1; i < q; ++i)
                for (int j = i; j > 0 && d2[j] < d2[j - 1]; --j) { int t = d2[j]; d2[j] = d2[j - 1]; d2[j - 1] = t; }
            for (int i = 0; i + 2 < q; ++i) ds += d2[i] * (q - 1 - i);
            heavy = ds > kCoreLight * 2;
        }
        if (mine && !heavy) venn_lane(li, false);
        unsigned hb = __ballot_sync(FULLMASK, heavy);
        while (hb) {                             // warp-cooperative raw histogram
            const int who = __ffs(hb) - 1;
            hb &= hb - 1;
            int a[FSGC_MAXQ], d[FSGC_MAXQ], pi_[FSGC_MAXQ];
            for (int bb = 0; bb < q; ++bb) {
                a[bb] = (int)s_leaf[who * FSGC_MAXC + P.anchor_pos[bb]];
                d[bb] = (int)(__ldg(G.offs + a[bb] + 1) - __ldg(G.offs + a[bb]));
                pi_[bb] = bb;
            }
            for (int i = 1; i < q; ++i)
                for (int j = i; j > 0 && d[pi_[j]] < d[pi_[j - 1]]; --j) { int t = pi_[j]; pi_[j] = pi_[j - 1]; pi_[j - 1] = t; }
            const bool pair_adj = q >= 2 && ((cadj[P.anchor_pos[pi_[q - 2]]] >> P.anchor_pos[pi_[q - 1]]) & 1);
            const int nscan = q >= 2 ? (pair_adj ? q - 2 : q - 1) : 0;
            for (int k = lane; k < V; k += 32) s_venn[who * V + k] = 0;
            __syncwarp();
            for (int i = 0; i < nscan; ++i) {
                const int64_t b0 = __ldg(G.offs + a[pi_[i]]);
                for (int s0 = 0; s0 < d[pi_[i]]; s0 += 32) {
                    const bool valid = s0 + lane < d[pi_[i]];
                    int m = 1 << i;
                    if (valid) {
                        const int x = __ldg(G.adj + b0 + s0 + lane);
                        for (int j = i + 1; j < q; ++j)
                            if (member(G, H, a[pi_[j]], x)) m |= 1 << j;
                    }
                    const unsigned act = __ballot_sync(FULLMASK, valid);
                    if (valid) {
                        const unsigned peers = __match_any_sync(act, m);
                        if (lane == __ffs(peers) - 1) s_venn[who * V + m] += __popc(peers);
                    }
                    __syncwarp();
                }
            }
            __syncwarp();
            if (lane == who) venn_lane(who, true);
            __syncwarp();
        }
        __syncwarp();
        if (VD.n && VD.warp) {                    // fc by the Venn term table, leaf by leaf
            for (int li = 0; li < cnt; ++li) {
                uint32_t vloc[1 << FSGC_MAXQ];
                for (int k = 0; k < V; ++k) vloc[k] = s_venn[li * V + k];
                venn_fc_warp<FSGC_FC_STACK>(vloc, q, P, VD, s_vrows[wib], lane, acc);
            }
        } else if (VD.n) {                        // small tables: a leaf per lane
            u128* rows = reinterpret_cast<u128*>(smem + kCoreWarps * 32 * (FSGC_MAXC + V));
            const bool mine = lane < cnt;
            uint32_t vloc[1 << FSGC_MAXQ];
            float bnd = 0.f;
            if (mine) {
                for (int k = 0; k < V; ++k) vloc[k] = s_venn[lane * V + k];
                bnd = venn_bound_log2(vloc, q, P) + VD.slack;
            }
            const bool all64 = __all_sync(FULLMASK, !mine || bnd < 55.f);
            if (mine && all64) {
                venn_terms_eval<uint64_t>(vloc, V, VD, (uint64_t*)(rows + threadIdx.x), 2 * blockDim.x, acc);
            } else if (mine && bnd < 119.f) {
                venn_terms_eval<u128>(vloc, V, VD, rows + threadIdx.x, blockDim.x, acc);
            } else if (mine) {
                for (int pi = 0; pi < nprog; ++pi) {
                    bool o = false;
                    const FringeProg fp = P.prog[pi];
                    const u128 f = fc_dispatch<FSGC_FC_STACK>(vloc, q, fp, o);
                    acc.add(fp.pat, f, o);
                }
            }
        }
        const int pairs = VD.n ? 0 : cnt * nprog;  // else fc over (leaf, program) pairs
        for (int tp = lane; tp < pairs; tp += 32) {
            const int l2 = tp / nprog, pi = tp - l2 * nprog;
            uint32_t vloc[1 << FSGC_MAXQ];
            for (int k = 0; k < V; ++k) vloc[k] = s_venn[l2 * V + k];
            bool o = false;
            u128 f;
            const int nt = __ldg(TD.cnt + pi);
            if (nt < 0 || !fc_partition(vloc, q, TD.terms + __ldg(TD.off + pi), nt, f)) {
                const FringeProg fp = P.prog[pi];
                f = fc_dispatch<FSGC_FC_STACK>(vloc, q, fp, o);
            }
            acc.add(P.prog[pi].pat, f, o);
        }
        if (lane == 0) nmatch += cnt;
        cnt = 0;
        __syncwarp();
    };

    auto leaf = [&]() {
#pragma unroll
        for (int j = 0; j < FSGC_MAXC; ++j)
            if (lane == j && j < p) s_leaf[cnt * FSGC_MAXC + j] = (uint32_t)emb[j];
        ++cnt;
        if (cnt == 32) flush();
    };

    auto init_level = [&](int l) {
        int piv = -1, best = 0x7fffffff;
#pragma unroll
        for (int j = 0; j < FSGC_MAXC; ++j)
            if (j < l && (P.back[l] >> j & 1) && edeg[j] < best) { best = edeg[j]; piv = j; }
        int64_t b = eoff[piv], e = eoff[piv] + edeg[piv];
        if (P.gt[l]) {
            int lb = -1;
#pragma unroll
            for (int j = 0; j < FSGC_MAXC; ++j)
                if (j < l && (P.gt[l] >> j & 1)) lb = max(lb, emb[j]);
            b += upper_bound(G.adj + b, (int)(e - b), lb);
        }
        cur[l] = b;
        endp[l] = e;
        pend[l] = 0;
        pivl[l] = piv;
    };

    const int64_t total = W.end - W.begin;
    for (;;) {
        unsigned long long jq = 0;
        if (lane == 0) jq = atomicAdd(queue, 1ull);
        jq = __shfl_sync(FULLMASK, jq, 0);
        const int64_t g = (int64_t)jq * W.nshards + W.shard;
        const int64_t t0 = g * W.chunk;
        if (t0 >= total) break;
        const int64_t t1 = min(t0 + (int64_t)W.chunk, total);
        for (int64_t t = t0; t < t1; ++t) {
            const int64_t item = W.end - 1 - t;   // heavy roots first
            int u0, u1;
            if (P.root_mode == ROOT_ORIENTED) { u0 = __ldg(G.osrc + item); u1 = __ldg(G.odst + item); }
            else { u0 = __ldg(G.row + item); u1 = __ldg(G.adj + item); }
            emb[0] = u0; eoff[0] = G.offs[u0]; edeg[0] = (int)(G.offs[u0 + 1] - eoff[0]);
            emb[1] = u1; eoff[1] = G.offs[u1]; edeg[1] = (int)(G.offs[u1 + 1] - eoff[1]);
            if (W.degfilter && (edeg[0] < P.mindeg[0] || edeg[1] < P.mindeg[1])) continue;
            int lvl = 2;
            init_level(2);
            while (lvl >= 2) {
                if (pend[lvl] == 0) {
                    if (cur[lvl] >= endp[lvl]) { --lvl; continue; }
                    const int64_t pidx = cur[lvl] + lane;
                    bool ok = pidx < endp[lvl];
                    const int x = ok ? __ldg(G.adj + pidx) : -1;
                    if (ok) {
#pragma unroll
                        for (int j = 0; j < FSGC_MAXC; ++j)
                            if (j < lvl && (x == emb[j] || ((P.gt[lvl] >> j & 1) && x <= emb[j]))) ok = false;
                    }
                    if (ok && W.degfilter) ok = (int)(G.offs[x + 1] - G.offs[x]) >= P.mindeg[lvl];
                    if (ok) {
                        const int piv = pivl[lvl];
                        for (int j = 0; j < lvl && ok; ++j)
                            if ((P.back[lvl] >> j & 1) && j != piv) ok = member(G, H, emb[j], x);
                    }
                    pend[lvl] = __ballot_sync(FULLMASK, ok);
                    cur[lvl] += 32;   // candidates are re-read from adj[cur - 32 + who]
                    continue;
                }
                const int who = __ffs(pend[lvl]) - 1;
                pend[lvl] &= pend[lvl] - 1;
                const int x = __ldg(G.adj + (cur[lvl] - 32) + who);
                emb[lvl] = x;
                eoff[lvl] = G.offs[x];
                edeg[lvl] = (int)(G.offs[x + 1] - eoff[lvl]);
                if (lvl == p - 1) {
                    leaf();
                } else {
                    ++lvl;
                    init_level(lvl);
                }
            }
        }
    }
    if (cnt) flush();
    block_publish<NP>(acc, nmatch, S);
}

// constant tables of THIS translation unit (every kernel TU has its own
// copies of the __constant__ / __device__ tables): the binomial table and the
// inverses of the odd parts of 1..63 mod 2^128 (Newton iteration)
static int dev_consts_init() {
    binom_table_init<<<1, 32>>>();
    if (cudaGetLastError() != cudaSuccess) return FSGC_ERR_CUDA;
    uint64_t inv[64] = {0}, invh[64] = {0};
    uint32_t tz[64] = {0};
    for (int t = 1; t < 64; ++t) {
        int z = 0;
        while (!((t >> z) & 1)) ++z;
        const u128 od = (u128)(t >> z);
        u128 x = od;
        for (int it = 0; it < 7; ++it) x *= (u128)2 - od * x;   // 3 -> 6 -> ... -> 384 correct bits
        inv[t] = u128_lo(x);
        invh[t] = u128_hi(x);
        tz[t] = (uint32_t)z;
    }
    if (cudaMemcpyToSymbol(c_inv_odd, inv, sizeof inv) != cudaSuccess) return FSGC_ERR_CUDA;
    if (cudaMemcpyToSymbol(c_inv_odd_hi, invh, sizeof invh) != cudaSuccess) return FSGC_ERR_CUDA;
    if (cudaMemcpyToSymbol(c_tz, tz, sizeof tz) != cudaSuccess) return FSGC_ERR_CUDA;
    return FSGC_OK;
}

}  // namespace
