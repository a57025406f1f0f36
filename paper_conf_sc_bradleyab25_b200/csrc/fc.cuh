// fc.cuh -- the fringe counting function on the device.
//
//   fc_eval<A>     iterative form of PAPER.md Listing 5 (Fig. 5) for any core
//   edge_formula<A> Sec. 3.1's closed form for 2-vertex cores (k tails on u,
//                  l tails on v, m wedge fringes) -- the paper's "specialized
//                  code" for small cores (Sec. 3.4); equal to Listing 5 on
//                  q = 2 diagrams (pinned in tests/test_oracle.py)
//
// Arithmetic policy A: Exact64 when the no-overflow bound holds, else the
// checked 128-bit path.  Bound: every product of binomials along a Listing 5
// path, every binomial intermediate r*(n-k+i) <= n^i, and the final sum are
// at most N^K, where N = size of the union of the anchors' external sets (the
// sum of all Venn entries) and K = total number of fringes; so
// bitlen(N) * K <= 63 implies everything fits in 64 bits.
#pragma once
#include "internal.h"
#include "u128.cuh"

// C(n, k) for n < kBinomN, k < kBinomK, filled once per device by
// fsgc_binom_table_init (entries that exceed 2^64 wrap; Exact64 never reads
// them because it only runs when N^K < 2^63, hence C(n, k) < 2^63)
constexpr int kBinomN = 2048, kBinomK = 8;
static __device__ uint64_t g_binom[kBinomN][kBinomK];   // (fc.cuh is included by count.cu only)

struct Exact64 {
    typedef uint64_t T;
    static constexpr bool is_wide = false;
    static __device__ __forceinline__ T add(T a, T b, bool&) { return a + b; }
    static __device__ __forceinline__ T mul(T a, T b, bool&) { return a * b; }
    static __device__ __forceinline__ T binom(uint64_t n, uint32_t k, bool&) {
        if (k > n) return 0;
        switch (k) {   // falling factorial / k!, exact division (no memory, no div)
            case 0: return 1;
            case 1: return n;
            case 2: return (n & 1) ? n * ((n - 1) >> 1) : (n >> 1) * (n - 1);
            case 3: return exact_div_const<6>(n * (n - 1) * (n - 2));
            case 4: return exact_div_const<24>(n * (n - 1) * (n - 2) * (n - 3));
            default: break;
        }
        if (n < (uint64_t)kBinomN && k < (uint32_t)kBinomK) return __ldg(&g_binom[n][k]);
        uint64_t r = 1;
        for (uint32_t i = 1; i <= k; ++i) r = exact_div(r * (n - k + i), i);
        return r;
    }
    template <uint32_t D>
    static __device__ __forceinline__ uint64_t exact_div_const(uint64_t x) {
        constexpr int tz = __builtin_ctz(D);
        constexpr uint64_t od = D >> tz;
        constexpr uint64_t i0 = od, i1 = i0 * (2 - od * i0), i2 = i1 * (2 - od * i1), i3 = i2 * (2 - od * i2),
                           i4 = i3 * (2 - od * i3), inv = i4 * (2 - od * i4);
        return (x >> tz) * inv;
    }
    // x / d for d | x (exact): shift out the 2-adic part, multiply by the
    // inverse of the odd part mod 2^64 (Newton: 5 steps from 3 correct bits)
    static __device__ __forceinline__ uint64_t exact_div(uint64_t x, uint32_t d) {
        const int tz = __ffs(d) - 1;
        x >>= tz;
        const uint64_t od = (uint64_t)(d >> tz);
        uint64_t inv = od;
#pragma unroll
        for (int it = 0; it < 5; ++it) inv *= 2 - od * inv;
        return x * inv;
    }
    static __device__ __forceinline__ u128 widen(T x) { return (u128)x; }
};

struct Checked128 {
    typedef u128 T;
    static constexpr bool is_wide = true;
    static __device__ __forceinline__ T add(T a, T b, bool& o) { return add_ovf(a, b, o); }
    static __device__ __forceinline__ T mul(T a, T b, bool& o) { return mul_ovf(a, b, o); }
    static __device__ __forceinline__ T binom(uint64_t n, uint32_t k, bool& o) { return binom_ovf(n, k, o); }
    static __device__ __forceinline__ u128 widen(T x) { return x; }
};

__device__ __forceinline__ int bitlen64(uint64_t x) { return 64 - __clzll((long long)x); }

// true if N^K < 2^63 (see header)
__device__ __forceinline__ bool fits64(uint64_t N, int K) { return (int64_t)bitlen64(N) * K <= 63; }

// Iterative Listing 5: the recursion fc(pos, rem, idx) with an explicit
// stack; `venn` (this lane's private copy) is decremented and restored as in
// lines 10/12 and 18/20 of the listing.
template <class A, int STACK>
__device__ typename A::T fc_eval(uint32_t* venn, int q, const FringeProg& P, bool& ovf) {
    typedef typename A::T T;
    const int s = P.s;
    if (s == 0) return (T)1;
    const int full = (1 << q) - 1;
    struct Fr { T M; uint32_t vc; uint8_t pos, rem, idx, i, top, kind; };
    Fr st[STACK];
    int sp = 0;
    T total = 0;
    int pos = 0, rem = P.k[0], idx = P.anch[0];
    T M = 1;
    for (;;) {
        for (;;) {                                       // enter fc(pos, rem, idx)
            if (rem == 0) {                              // line 6: next fringe type
                if (++pos == s) { total = A::add(total, M, ovf); break; }   // line 5
                rem = P.k[pos];
                idx = P.anch[pos];
                continue;
            }
            const uint32_t vc = venn[idx];               // line 7
            if (idx == full) {                           // line 8: last entry
                if ((uint32_t)rem > vc) break;           // line 9: no solution
                M = A::mul(M, A::binom(vc, (uint32_t)rem, ovf), ovf);      // line 11
                venn[idx] = vc - rem;                    // line 10
                Fr f;
                f.kind = 0; f.idx = (uint8_t)idx; f.rem = (uint8_t)rem;
                st[sp++] = f;
                rem = 0;
                continue;
            }
            const int top = min(rem, (int)vc);           // line 16
            Fr f;
            f.M = M; f.vc = vc; f.pos = (uint8_t)pos; f.rem = (uint8_t)rem;
            f.idx = (uint8_t)idx; f.i = 0; f.top = (uint8_t)top; f.kind = 1;
            st[sp++] = f;                                // i = 0: C(vc, 0) = 1
            idx = (idx + 1) | P.anch[pos];               // line 19: next covering entry
        }
        for (;;) {                                       // return: undo + advance
            if (sp == 0) return total;
            Fr& f = st[sp - 1];
            if (f.kind == 0) { venn[f.idx] += f.rem; --sp; continue; }     // line 12
            venn[f.idx] += f.i;                          // line 20
            if (++f.i > f.top) { --sp; continue; }
            venn[f.idx] -= f.i;                          // line 18
            M = A::mul(f.M, A::binom(f.vc, f.i, ovf), ovf);
            pos = f.pos;
            rem = f.rem - f.i;
            idx = (f.idx + 1) | P.anch[f.pos];
            break;
        }
    }
}

// fc for one (diagram, program): 64-bit when the bound allows, else 128.
template <int STACK>
__device__ __forceinline__ u128 fc_dispatch(uint32_t* venn, int q, const FringeProg& P, bool& ovf) {
    uint64_t N = 0;
    for (int e = 1; e < (1 << q); ++e) N += venn[e];
    if (fits64(N, P.ksum)) {
        bool dummy = false;
        return (u128)fc_eval<Exact64, STACK>(venn, q, P, dummy);
    }
    return fc_eval<Checked128, STACK>(venn, q, P, ovf);
}

// Sec. 3.1, last displayed formula: k tails on u, l tails on v, m wedges;
// nu = |e(u) \ e(v)|, nv = |e(v) \ e(u)|, nuv = |e(u) & e(v)|.
template <class A>
__device__ __forceinline__ typename A::T edge_formula(uint64_t nu, uint64_t nv, uint64_t nuv, int k, int l, int m,
                                                      bool& ovf) {
    typedef typename A::T T;
    T tot = 0;
    if ((uint64_t)m > nuv) return tot;
    const int imax = (int)min((uint64_t)k, nuv);
    for (int i = 0; i <= imax; ++i) {
        if ((uint64_t)(k - i) > nu) continue;
        const T a = A::mul(A::binom(nu, k - i, ovf), A::binom(nuv, i, ovf), ovf);
        const uint64_t r1 = nuv - i;
        const int jmax = (int)min((uint64_t)l, r1);
        for (int j = 0; j <= jmax; ++j) {
            if ((uint64_t)(l - j) > nv || (uint64_t)m > r1 - j) continue;
            T b = A::mul(A::binom(nv, l - j, ovf), A::binom(r1, j, ovf), ovf);
            b = A::mul(b, A::binom(r1 - j, m, ovf), ovf);
            tot = A::add(tot, A::mul(a, b, ovf), ovf);
        }
    }
    return tot;
}
