// listing.cuh -- triangle listing from the MIDDLE vertex (included by
// count.cu): the per-edge support pass and the triangle-core pass share it.
//
// PAPER.md Sec. 3.6 intersects the neighbour lists of the matched vertices
// per core match; Sec. 3.3 needs, per triangle core (u, v, w), the sizes of
// the Venn regions of e(u), e(v), e(w).  Here every triangle a < b < c
// (degree-ordered ids, Sec. 3.1 symmetry breaking) is found from its middle
// vertex b: c in N+(a) & N+(b) with a in N-(b) = {a < b, a ~ b} and c > b.
// A work unit is (b, slice of N-(b)); N+(b) is staged in a shared-memory
// hash table once per b, and for every in-neighbour a of the slice the tail
// of N+(a) after b (b's position in N+(a) comes from graph.rev) is streamed
// through the table.  Work: sum_a out(a)^2 / 2 probes, coalesced tail reads,
// no per-match binary search.
//
//   warp tables  (out(b) <= capw = 256, the many small middles): one warp per
//                unit with its own table; the slice's tails are concatenated
//                (warp prefix sum) so the 32 lanes read 32 consecutive
//                virtual elements whatever the tail lengths;
//   block tables (out(b) > capw, the heavy middles: RMAT-26 has out(b) up to
//                3,004): one block per unit with a table sized to the graph's
//                largest out(b); the warps take 32 in-neighbours at a time
//                from a block-local counter (dynamic within the block) and
//                stream one tail at a time, kILP loads in flight per lane.
// Units come from a global atomic queue (heavy middles first for the block
// kernel), dealt round-robin over the shards of a multi-GPU count.
//
// Two visitors of the same listing (template flag TRI):
//   support   (TRI = false): c(e) = |N(u) & N(v)| for every oriented edge:
//             a hit (a, b, c) adds 1 to c(bc) (shared counter per table slot,
//             flushed when the table changes), c(ac) (global reduction) and
//             c(ab) (ballot count per in-neighbour, one add per (a, b));
//   tri-core  (TRI = true, after the support pass): a hit is a triangle core
//             match (u, v, w) = (a, b, c); its degrees and supports are
//             gathered (deg / c(bc) of the N+(b) entries are staged beside
//             the table), buffered per warp, and the buffer is flushed
//             through the Venn diagram (Sec. 3.3) and the fringe counting
//             function (Venn term table, else Listing 5).

#ifndef FSGC_ZONLY_MINB
#define FSGC_ZONLY_MINB 4         // resident blocks per SM the Z-only listing kernels are compiled for
#endif
constexpr int kLeafCap = 64;      // leaf buffer per warp (flushed at >= 32)
constexpr int kLeafW = 9;         // a, b, c, du, dv, dw, cuv, e(ac), cvw
constexpr int kILP = 4;           // tail loads in flight per lane (block tables)
constexpr int kWarpTabWarps = 8;  // warps per block, warp-table kernels
constexpr int kBlockTabWarps = 16;   // warps per block, block-table support kernel
constexpr int kBlockTriWarps = 8;    // warps per block, block-table tri-core kernel (MODE 1)
constexpr int kBlockTriWarpsMax = 12;   // Z-only block kernel: 8 or 12 warps (host: most resident warps);
                                        // compiled for 2 blocks of 12 warps: up to 80 registers, no spills
constexpr int kSubCSup = 512;        // in-entries per concatenated sub-chunk, block-table support kernel
constexpr int kSubCTri = 256;        // ... tri-core kernel (shared memory: 2 blocks/SM with RMAT-26's table)

__device__ __forceinline__ uint32_t hslot(int x, int hbits) { return ((uint32_t)x * 0x9E3779B1u) >> (32 - hbits); }

// slot of x in the table, -1 if absent (open addressing, linear probing)
__device__ __forceinline__ int hfind(const int32_t* key, int x, int hbits) {
    const uint32_t hm = (1u << hbits) - 1;
    uint32_t h = hslot(x, hbits);
    int y;
    while ((y = key[h]) != x && y != -1) h = (h + 1) & hm;
    return y == x ? (int)h : -1;
}

// the table of N+(b): keys, kpos = position of the key in N+(b), and the
// payload, built by `nthr` threads (a warp or a block; the caller
// synchronises before and after).  Support: cnt[i] = 0 (the c(b, x)
// counters, by position in N+(b)).  Tri-core: tsup[i] = c(b, x), tdeg[i] = deg(x) for the i-th
// entry x of N+(b).
template <bool TRI>
__device__ __forceinline__ void table_build(const GraphDev& G, const OrientDev& O, const int* __restrict__ sup,
                                            int b, int64_t sb, int ob, int hbits, int32_t* key, int16_t* kpos,
                                            int32_t* cnt, int32_t* tsup, int32_t* tdeg, int tid, int nthr) {
    const uint32_t hm = (1u << hbits) - 1;
    const int64_t ob0 = TRI ? __ldg(O.oofs + b) : 0;
    for (int i = tid; i < ob; i += nthr) {
        const int x = __ldg(G.adj + sb + i);
        uint32_t h = hslot(x, hbits);
        while (atomicCAS(&key[h], -1, x) != -1) h = (h + 1) & hm;
        kpos[h] = (int16_t)i;
        if (TRI) {
            tsup[i] = __ldg(sup + ob0 + i);
            tdeg[i] = (int)(__ldg(G.offs + x + 1) - __ldg(G.offs + x));
        } else {
            cnt[i] = 0;
        }
    }
}

// support: add the table's c(b, x) counters (by position in N+(b)) to the
// support array -- the edges (b, x) are consecutive oriented indices
__device__ __forceinline__ void table_flush(const OrientDev& O, int* __restrict__ sup, int b, int ob,
                                            const int32_t* cnt, int tid, int nthr) {
    const int64_t base = __ldg(O.oofs + b);
    for (int i = tid; i < ob; i += nthr)
        if (cnt[i]) atomicAdd(sup + base + i, cnt[i]);
}

// ------------------------------------------------------------------------
// tri-core visitor: the per-warp leaf buffer and its flush
struct TriCtx {
    int q, V, nprog;
    int proj[8];        // core position mask F (bit0 u, bit1 v, bit2 w) -> Venn bit mask
    bool need_t;        // the anchors' Venn needs t = |N(u) & N(v) & N(w)|
    int mindeg0, mindeg1, mindeg2;
    int degfilter;
    int cmask[8];       // Venn bit mask -> core position mask (bit0 u, bit1 v, bit2 w)
};

// Necessary condition for fc > 0 from the pairwise quantities alone: some
// program whose every fringe type t' fits k_t' <= Z[A_t'] -- with
// Z[{x}] = deg(x) - 2 and Z[{x, y}] = c(xy) - 1 exact (core vertices
// excluded) and Z[{u, v, w}] = t <= min c(..) - 1.  Leaves that fail it have
// fc = 0 for every program: no triple intersection, no fc evaluation.
__device__ __forceinline__ bool tri_alive(const CoreProg& P, const TriCtx& C, int du, int dv, int dw, int cuv,
                                          int cuw, int cvw) {
    int z[8];
    z[0] = 1 << 30;
    z[1] = du - 2; z[2] = dv - 2; z[4] = dw - 2;
    z[3] = cuv - 1; z[5] = cuw - 1; z[6] = cvw - 1;
    z[7] = min(z[3], min(z[5], z[6]));
    for (int pi = 0; pi < C.nprog; ++pi) {
        const FringeProg& fp = P.prog[pi];
        bool ok = true;
        for (int t = 0; t < fp.s && ok; ++t) ok = (int)fp.k[t] <= z[C.cmask[fp.anch[t]]];
        if (ok) return true;
    }
    return C.nprog == 0;
}

__device__ __forceinline__ void tri_ctx_init(TriCtx& C, const CoreProg& P, const WorkDesc& W) {
    C.q = P.q;
    C.V = 1 << P.q;
    C.nprog = P.nprog;
#pragma unroll
    for (int F = 0; F < 8; ++F) {
        int M = 0;
        for (int b = 0; b < P.q; ++b)
            if ((F >> P.anchor_pos[b]) & 1) M |= 1 << b;
        C.proj[F] = M;
    }
#pragma unroll
    for (int M = 0; M < 8; ++M) {
        int cm = 0;
        for (int b = 0; b < P.q; ++b)
            if ((M >> b) & 1) cm |= 1 << P.anchor_pos[b];
        C.cmask[M] = cm;
    }
    // Does any program's fc depend on t = |N(u) & N(v) & N(w)|?  A vertex of
    // region F (core positions it is adjacent to) can serve the fringe types
    // t' with A_t' inside proj[F] -- its signature.  A program's fc depends
    // only on the sizes of its signature classes (vertices with the same
    // signature are interchangeable), and t enters region F with sign +1
    // (|F| odd) or -1 (|F| = 2).  So t is needed iff some program has a
    // non-empty signature class whose signs do not cancel (e.g. a
    // tri-fringe, or tails on all three core vertices); otherwise any t in
    // the feasible range gives the same fc (tri_flush takes the smallest).
    C.need_t = false;
    for (int pi = 0; pi < P.nprog && !C.need_t; ++pi) {
        const FringeProg& fp = P.prog[pi];
        int sig[8], coef[8];
        for (int F = 1; F < 8; ++F) {
            int sg = 0;
            for (int t = 0; t < fp.s; ++t)
                if ((C.proj[F] & fp.anch[t]) == fp.anch[t]) sg |= 1 << t;
            sig[F] = sg;
            coef[F] = 0;
        }
        for (int F = 1; F < 8; ++F) {
            if (!sig[F]) continue;
            int c = 0;
            for (int G = 1; G < 8; ++G)
                if (sig[G] == sig[F]) c += (__popc(G) & 1) ? 1 : -1;
            if (c != 0) C.need_t = true;
        }
    }
    C.mindeg0 = P.mindeg[0];
    C.mindeg1 = P.mindeg[1];
    C.mindeg2 = P.mindeg[2];
    C.degfilter = W.degfilter;
}

template <class W>
__device__ __forceinline__ W sext(int64_t c);
template <>
__device__ __forceinline__ uint64_t sext<uint64_t>(int64_t c) { return (uint64_t)c; }
template <>
__device__ __forceinline__ u128 sext<u128>(int64_t c) { return (u128)(__int128)c; }

// C(n, j) mod 2^bits(W) by the exact-division chain C(n, i) = C(n, i-1) (n-i+1) / i
// (division by the odd part of i via its inverse, by the 2-power by a shift);
// exact when C(n, i) * i fits for every i <= j -- the tier bound of the caller
template <class W>
__device__ __forceinline__ W binom_fly(uint64_t n, int j) {
    W c = (W)n;
    for (int i = 2; i <= j; ++i) c = ((c * (W)(n - (uint64_t)i + 1)) >> c_tz[i]) * inv_odd(i, c);
    return c;
}
// 64-bit tier, the common small case: j <= 4 and n < 2^16 by the products
// n(n-1)(n-2)(n-3) < 2^64 in 32-bit pieces and one exact division (a shift
// for the 2-power, the inverse of 3 mod 2^64 for the odd part); the factors
// vanish for n < j as in the chain
template <>
__device__ __forceinline__ uint64_t binom_fly<uint64_t>(uint64_t n, int j) {
    if (n < 65536u && j <= 4) {
        const uint32_t m = (uint32_t)n;
        const uint32_t a = m * (m - 1u);                     // < 2^32
        if (j <= 1) return j == 1 ? n : 1u;
        if (j == 2) return a >> 1;
        const uint64_t inv3 = 0xAAAAAAAAAAAAAAABull;
        if (j == 3) return (((uint64_t)a * (uint64_t)(m - 2u)) >> 1) * inv3;
        return (((uint64_t)a * (uint64_t)(uint32_t)((m - 2u) * (m - 3u))) >> 3) * inv3;
    }
    uint64_t c = n;
    for (int i = 2; i <= j; ++i) c = ((c * (n - (uint64_t)i + 1)) >> c_tz[i]) * c_inv_odd[i];
    return c;
}

// one pattern's terms [t0, t1) of the Z-term table on one triangle, mod
// 2^bits(W).  Out of line: one copy per tier, called once per (leaf, pattern)
template <class W>
__device__ __noinline__ W zterm_sum(const int* z, const ZTerm* zt, int t0, int t1) {
    // z: the leaf's Z values by core mask in the thread's local memory (one
    // load per factor at a warp-uniform index instead of a select chain)
    W sum = 0;
    for (int t = t0; t < t1; ++t) {
        const uint4 e = *reinterpret_cast<const uint4*>(zt + t);   // shared (staged) or global
        W pr = sext<W>((int64_t)(((uint64_t)e.y << 32) | e.x));
        const int nf = (e.z >> 8) & 255;
        uint64_t codes = (uint64_t)(e.z >> 16) | ((uint64_t)e.w << 16);   // 8-bit factor codes
        for (int i = 0; i < nf; ++i, codes >>= 8) {
            const int code = (int)(codes & 255);
            pr *= binom_fly<W>((uint64_t)z[code >> 5], code & 31);
        }
        sum += pr;
    }
    return sum;
}

// the Z-term table on the warp's 32 triangle leaves (z[cm] = Z of the
// core-position set cm), arithmetic mod 2^64 or 2^128 per pattern (the host's
// per-pattern threshold on the leaf's largest degree: the binomials times j
// and the pattern's per-leaf sum fit 64 bits; else 128 bits, which the
// kernel's global bound guarantees).  Terms are grouped by pattern; each pattern's per-leaf sums
// are reduced over the warp (shuffles) and lane 0 adds the total to the warp's
// shared accumulator.  No binomial rows are kept.  Warp-uniform call.
// the pass's Z-term table staged in shared memory at kernel start (the flush
// is out of line, so reading it from the kernel parameters would go through
// generic loads)
constexpr int kZShared = 64;
struct ZShared {
    const ZTerm* terms;          // shared copy (or the global table when it is larger)
    const uint16_t* zoff;        // [FSGC_MAXPATS + 1]
    const int32_t* z64;          // [FSGC_MAXPATS]
};

// warp sum of a non-negative value below 2^(16 * limbs): the 16-bit limbs
// are summed with __reduce_add_sync (each limb sum < 2^21), then recombined --
// a handful of REDUX instead of a 5-round 128-bit shuffle tree
template <int LIMBS>
__device__ __forceinline__ u128 warp_sum_limbs(u128 v) {
    u128 tot = 0;
#pragma unroll
    for (int l = 0; l < LIMBS; ++l) {
        const unsigned part = __reduce_add_sync(FULLMASK, (unsigned)((uint64_t)(v >> (16 * l)) & 0xffffu));
        tot += (u128)part << (16 * l);
    }
    return tot;
}

template <int NP, bool ZONLY>
__device__ __forceinline__ void zterms_eval_warp(bool act, int zmax, const int (&z)[8], const ZShared& T,
                                                 const SAcc& sa, int lane) {
    // (a runtime pattern loop: the accumulators are in shared memory, so the
    // code is not replicated per pattern)
#pragma unroll 1
    for (int p = 0; p < NP; ++p) {
        const int t0 = T.zoff[p], t1 = T.zoff[p + 1];
        if (t0 == t1) continue;
        // the tier per pattern (warp-uniform): 64-bit unless some leaf's
        // largest degree exceeds the pattern's 64-bit threshold (then the
        // per-leaf sum is below 2^119 by the kernel's bound)
        u128 tot;
        if (__all_sync(FULLMASK, !act || zmax <= T.z64[p])) {
            const uint64_t v = act ? zterm_sum<uint64_t>(z, T.terms, t0, t1) : 0;
            tot = warp_sum_limbs<4>((u128)v);      // 32 x < 2^62: the sum fits 67 bits
        } else {
            const u128 v = act ? zterm_sum<u128>(z, T.terms, t0, t1) : 0;
            tot = warp_sum_limbs<8>(v);            // 32 x < 2^119 < 2^128
        }
        if (lane == 0 && tot != 0) {
            if (ZONLY) {   // only this lane writes the warp's sums: a plain 128-bit add
                AccDev& d = sa.a[p];
                const u128 old = u128_make(d.lo, d.hi);
                const u128 nw = old + tot;
                d.lo = u128_lo(nw);
                d.hi = u128_hi(nw);
                if (nw < old) d.ovf = 1;
            } else {       // the Venn / Listing 5 lanes of this warp add atomically
                atomic_add_u128(sa.a + p, tot, false);
            }
        }
    }
}

// Flush the warp's `cnt` buffered triangle matches (leaf[i * kLeafW + .]):
// Venn diagram (Sec. 3.3) -- with c(xy) = |N(x) & N(y)| and
// t = |N(u) & N(v) & N(w)| the 7 regions of e(u), e(v), e(w) (core vertices
// excluded; each core vertex is adjacent to the other two) are
//   uvw = t, uv = c(uv) - 1 - t, uw = c(uw) - 1 - t, vw = c(vw) - 1 - t,
//   u = deg(u) - 2 - uv - uw - t (likewise v, w),
// projected onto the q anchors -- then fc (Venn term table in the 64- or
// 128-bit tier, else Listing 5 per program).  t by one triple intersection:
// N(u), the shortest list (u has the lowest degree), scanned against N(v),
// N(w) through hub bitmaps or galloping cursors; warp-cooperative for long
// lists.
__device__ __noinline__ void tri_fc_venn(const CoreProg& P, const VennDev& VD, const TriCtx& C, bool alive, bool zfb,
                                         int t, int du, int dv, int dw, int cuv, int cuw, int cvw, u128* lane_rows,
                                         int lane_stride, u128* warp_rows, int lane, const SAcc acc);

template <int NP, bool ZONLY>
__device__ __noinline__ void tri_flush(const GraphDev& G, const HubDev& H, const CoreProg& P, const VennDev& VD,
                                       const TriCtx& C, const int* __restrict__ sup, uint32_t* leaf, int cnt,
                                       u128* lane_rows, int lane_stride, u128* warp_rows, int lane, const SAcc sa,
                                       const ZShared ZS) {
    __syncwarp();
    for (int base = 0; base < cnt; base += 32) {
        const int li = base + lane;
        const bool mine = li < cnt;
        const uint32_t* L = leaf + li * kLeafW;
        int lu = 0, lv = 0, lw = 0, du = 0, dv = 0, dw = 0, cuv = 0, cuw = 0, cvw = 0, t = 0;
        if (mine) {
            lu = (int)L[0]; lv = (int)L[1]; lw = (int)L[2];
            du = (int)L[3]; dv = (int)L[4]; dw = (int)L[5];
            cuv = (int)L[6]; cvw = (int)L[8];
            cuw = __ldg(sup + L[7]);
        }
        // leaves whose fc is 0 for every program (necessary condition from
        // degrees and supports) are counted as matches and skipped
        // (the Z-term path without t evaluates every leaf: cheaper than the test)
        const bool alive = mine && ((VD.zn && !VD.zneed7) || tri_alive(P, C, du, dv, dw, cuv, cuw, cvw));
        // Z-term path: tier bound from the largest Z in use and the largest
        // program (prod_t C(Z_t, k_t) <= Zmax^K); past 2^119 the leaf takes
        // the checked Listing 5 on its Venn diagram
        const int zmax = max(max(du, dv), dw);   // >= every Z of the leaf
        const bool zfb = !ZONLY && VD.zn && alive && zmax > VD.zmax128;
        const bool want_t = alive && (VD.zn ? (VD.zneed7 || (zfb && C.need_t)) : C.need_t);
        const bool heavy = want_t && du > 32;
        if (want_t && !heavy) {
            Cursor cv, cw;
            cv.init(G, H, lv);
            cw.init(G, H, lw);
            const int64_t b0 = __ldg(G.offs + lu);
            for (int i = 0; i < du; ++i) {
                const int x = __ldg(G.adj + b0 + i);
                if (cv.has(x) && cw.has(x)) ++t;
            }
        }
        unsigned hb = __ballot_sync(FULLMASK, heavy);
        while (hb) {
            const int who = __ffs(hb) - 1;
            hb &= hb - 1;
            const int hu = __shfl_sync(FULLMASK, lu, who), hv = __shfl_sync(FULLMASK, lv, who);
            const int hw = __shfl_sync(FULLMASK, lw, who), hd = __shfl_sync(FULLMASK, du, who);
            const int64_t b0 = __ldg(G.offs + hu);
            int tt = 0;
            for (int s0 = 0; s0 < hd; s0 += 32) {
                bool hit = false;
                if (s0 + lane < hd) {
                    const int x = __ldg(G.adj + b0 + s0 + lane);
                    hit = member(G, H, hv, x) && member(G, H, hw, x);
                }
                tt += __popc(__ballot_sync(FULLMASK, hit));
            }
            if (lane == who) t = tt;
        }
        if (alive && !want_t) {   // any feasible t: the smallest keeps every region >= 0
            t = max(max(0, cuv + cuw - du), max(cuv + cvw - dv, cuw + cvw - dw));
        }
        if (VD.zn) {                   // fc from the Z values (no Venn diagram)
            int z[8];
            z[0] = 0;
            z[1] = du - 2; z[2] = dv - 2; z[4] = dw - 2;
            z[3] = cuv - 1; z[5] = cuw - 1; z[6] = cvw - 1;
            z[7] = t;
            zterms_eval_warp<NP, ZONLY>(alive && !zfb, zmax, z, ZS, sa, lane);
            if (!__any_sync(FULLMASK, alive && zfb)) continue;
        }
        if constexpr (!ZONLY)
            tri_fc_venn(P, VD, C, alive, zfb, t, du, dv, dw, cuv, cuw, cvw, lane_rows, lane_stride, warp_rows, lane,
                        sa);
    }
    __syncwarp();
}

// the Venn-diagram part of the flush (out of line: not fetched on the Z-term
// path): Venn term table (per lane or per warp), else checked Listing 5
__device__ __noinline__ void tri_fc_venn(const CoreProg& P, const VennDev& VD, const TriCtx& C, bool alive, bool zfb,
                                         int t, int du, int dv, int dw, int cuv, int cuw, int cvw, u128* lane_rows,
                                         int lane_stride, u128* warp_rows, int lane, const SAcc acc) {
        uint32_t vq[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        if (alive) {
            int R[8];
            R[0] = 0;
            R[7] = t;
            R[3] = cuv - 1 - t;
            R[5] = cuw - 1 - t;
            R[6] = cvw - 1 - t;
            R[1] = du - 2 - R[3] - R[5] - t;
            R[2] = dv - 2 - R[3] - R[6] - t;
            R[4] = dw - 2 - R[5] - R[6] - t;
#pragma unroll
            for (int F = 1; F < 8; ++F)
                if (C.proj[F]) vq[C.proj[F]] += (uint32_t)R[F];
        }
        if (VD.zn) {                    // Z mode, fallback lanes: checked Listing 5
            if (alive && zfb)
                for (int pi = 0; pi < C.nprog; ++pi) {
                    const FringeProg fp = P.prog[pi];
                    bool o = false;
                    const u128 f = fc_dispatch<kTriStack>(vq, C.q, fp, o);
                    acc.add(fp.pat, f, o);
                }
        } else if (VD.n && VD.warp) {          // one diagram per warp, lanes over the terms
            unsigned am = __ballot_sync(FULLMASK, alive);
            while (am) {
                const int l = __ffs(am) - 1;
                am &= am - 1;
                uint32_t vloc[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) vloc[k] = __shfl_sync(FULLMASK, vq[k], l);
                venn_fc_warp<kTriStack>(vloc, C.q, P, VD, warp_rows, lane, acc);
            }
        } else if (VD.n) {              // one diagram per lane, rows per thread
            float bnd = 0.f;
            if (alive) bnd = venn_bound_log2(vq, C.q, P) + VD.slack;
            const bool all64 = __all_sync(FULLMASK, !alive || bnd < 55.f);
            if (alive && all64) {
                venn_terms_eval<uint64_t>(vq, C.V, VD, (uint64_t*)lane_rows, 2 * lane_stride, acc);
            } else if (alive && bnd < 119.f) {
                venn_terms_eval<u128>(vq, C.V, VD, lane_rows, lane_stride, acc);
            } else if (alive) {
                for (int pi = 0; pi < C.nprog; ++pi) {
                    const FringeProg fp = P.prog[pi];
                    bool o = false;
                    const u128 f = fc_dispatch<kTriStack>(vq, C.q, fp, o);
                    acc.add(fp.pat, f, o);
                }
            }
        } else {                        // Listing 5 per program (no table)
            if (alive)
                for (int pi = 0; pi < C.nprog; ++pi) {
                    const FringeProg fp = P.prog[pi];
                    bool o = false;
                    const u128 f = fc_dispatch<kTriStack>(vq, C.q, fp, o);
                    acc.add(fp.pat, f, o);
                }
        }
}

// stage the Z-term table of the pass in shared memory (block-wide, the caller
// synchronises)
__device__ __forceinline__ ZShared zshared_stage(const VennDev& VD, ZTerm* s_zt, uint16_t* s_zoff, int32_t* s_z64,
                                                 int tid, int nthr) {
    const bool fits = VD.zn <= kZShared;
    if (fits)
        for (int i = tid; i < VD.zn; i += nthr) s_zt[i] = VD.zterms[i];
    for (int i = tid; i <= FSGC_MAXPATS; i += nthr) s_zoff[i] = VD.zoff[i];
    for (int i = tid; i < FSGC_MAXPATS; i += nthr) s_z64[i] = VD.zmax64p[i];
    return ZShared{fits ? s_zt : VD.zterms, s_zoff, s_z64};
}

// end of a triangle-core kernel: the warps' shared pattern sums and match
// counts summed by warp 0, one 128-bit atomic per pattern into the pass
// result (the triangle-core sink is always in atomic mode)
template <int NP>
__device__ __forceinline__ void sacc_publish(AccDev (*s_acc)[NP], unsigned long long* s_nm, int nwb,
                                             unsigned long long nmatch, const Sink& S, int w, int lane) {
    if (lane == 0) s_nm[w] = nmatch;
    __syncthreads();
    if (w != 0) return;
    for (int p = lane; p < NP; p += 32) {
        u128 v = 0;
        bool o = false;
        for (int q = 0; q < nwb; ++q) {
            v = add_ovf(v, u128_make(s_acc[q][p].lo, s_acc[q][p].hi), o);
            o = o || s_acc[q][p].ovf;
        }
        if (v != 0 || o) atomic_add_u128(S.acc + p, v, o);
    }
    if (lane == 0) {
        unsigned long long nm = 0;
        for (int q = 0; q < nwb; ++q) nm += s_nm[q];
        if (nm) atomicAdd(S.matches, nm);
    }
}

// the warp's shared pattern sums as lane 0's register accumulators (for the
// block reduction at the end of a kernel)
template <int NP>
__device__ __forceinline__ AccN<NP> sacc_to_lane0(const AccDev* a, int lane) {
    __syncwarp();
    AccN<NP> A;
    A.init();
    if (lane == 0) {
#pragma unroll
        for (int p = 0; p < NP; ++p) {
            A.v[p] = u128_make(a[p].lo, a[p].hi);
            if (a[p].ovf) A.ovf |= 1u << p;
        }
    }
    return A;
}

// append the hits of one round (hit: this lane's candidate c is in N+(b)) to
// the warp's leaf buffer; the caller flushes at >= 32
__device__ __forceinline__ int tri_append(uint32_t* leaf, int cnt, bool hit, int a, int b, int c, int du, int dv,
                                          int dw, int cuv, uint32_t eac, int cvw, int lane) {
    const unsigned fm = __ballot_sync(FULLMASK, hit);
    if (hit) {
        uint32_t* L = leaf + (cnt + __popc(fm & ((1u << lane) - 1))) * kLeafW;
        L[0] = (uint32_t)a; L[1] = (uint32_t)b; L[2] = (uint32_t)c;
        L[3] = (uint32_t)du; L[4] = (uint32_t)dv; L[5] = (uint32_t)dw;
        L[6] = (uint32_t)cuv; L[7] = eac; L[8] = (uint32_t)cvw;
    }
    return cnt + __popc(fm);
}

// ------------------------------------------------------------------------
// warp-table kernel.  Shared memory per warp: table (key, kpos/cnt or
// tsup/tdeg: HS = 2 * FSGC_SUP_CAPW slots), slice arrays, leaf buffer (TRI)
constexpr int kWSub = 64;    // in-entries per half-slice of a warp unit (FSGC_SUP_SEG = 2 halves)
template <int MODE>
struct WarpTabLayout {
    static constexpr bool TRI = MODE != 0;
    static constexpr int HS = 2 * FSGC_SUP_CAPW;
    static constexpr size_t key_b = (size_t)HS * 4;
    static constexpr size_t kpos_b = (size_t)HS * 2;
    static constexpr size_t pay_b = TRI ? (size_t)FSGC_SUP_CAPW * 8 : (size_t)FSGC_SUP_CAPW * 4;   // tsup+tdeg | cnt
    static constexpr size_t slice_b = (size_t)(kWSub + 4) * 4 + (size_t)5 * kWSub * 4;
    static constexpr size_t leaf_b = TRI ? (size_t)kLeafCap * kLeafW * 4 : 0;
    static constexpr size_t rows_b = MODE == 1 ? (size_t)kMaxVennRows * 16 : 0;     // warp-mode term rows
    static constexpr size_t warp_b = key_b + kpos_b + pay_b + slice_b + leaf_b + rows_b;
    static constexpr size_t bytes = kWarpTabWarps * warp_b;
};

// MODE: 0 support pass, 1 triangle-core pass (every fc path), 2 triangle-core
// pass on the Z-term path only (the host picks it when no leaf can leave the
// 128-bit tier: no Venn / Listing 5 code in the kernel, fewer registers)
template <int MODE, int NP>
__global__ void __launch_bounds__(kWarpTabWarps * 32, MODE == 2 ? FSGC_ZONLY_MINB : MODE + 1) list_warp_kernel(
    GraphDev G, OrientDev O, HubDev H, const int32_t* __restrict__ rev, const uint64_t* __restrict__ units,
    int64_t nunits, int* __restrict__ sup, unsigned long long* queue, int shard, int nshards, const __grid_constant__ CoreProg P,
    WorkDesc W, const __grid_constant__ VennDev VD, const Sink S) {
    constexpr bool TRI = MODE != 0;
    typedef WarpTabLayout<MODE> Lay;
    extern __shared__ __align__(16) unsigned char s_lw[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    unsigned char* tb = s_lw + (size_t)w * Lay::warp_b;
    int32_t* key = reinterpret_cast<int32_t*>(tb);
    int16_t* kpos = reinterpret_cast<int16_t*>(tb + Lay::key_b);
    int32_t* pay0 = reinterpret_cast<int32_t*>(tb + Lay::key_b + Lay::kpos_b);   // cnt[slot] | tsup[pos]
    int32_t* pay1 = pay0 + FSGC_SUP_CAPW;                                         // - | tdeg[pos]
    unsigned char* wb = tb + Lay::key_b + Lay::kpos_b + Lay::pay_b;
    int32_t* pre = reinterpret_cast<int32_t*>(wb);                           // [kWSub + 4]
    uint32_t* q0 = reinterpret_cast<uint32_t*>(wb + (kWSub + 4) * 4);        // tail start per in-entry
    uint32_t* da = q0 + kWSub;                                               // split[a] - oofs[a]
    int32_t* ea = reinterpret_cast<int32_t*>(da + kWSub);                    // e(ab) | a
    int32_t* xa = ea + kWSub;                                                // c(ab) count | deg a
    int32_t* ya = xa + kWSub;                                                // - | c(ab)
    uint32_t* leaf = reinterpret_cast<uint32_t*>(wb + Lay::slice_b);
    u128* wrows = reinterpret_cast<u128*>(wb + Lay::slice_b + Lay::leaf_b);
    u128* lrows = reinterpret_cast<u128*>(s_lw + Lay::bytes) + threadIdx.x;  // lane-mode term rows

    __shared__ AccDev s_acc[kWarpTabWarps][TRI ? NP : 1];   // per-warp pattern sums (tri-core)
    __shared__ ZTerm s_zt[TRI ? kZShared : 1];
    __shared__ uint16_t s_zoff[FSGC_MAXPATS + 1];
    __shared__ int32_t s_z64[FSGC_MAXPATS];
    const SAcc sa{s_acc[w]};
    if (TRI && lane < NP) s_acc[w][lane] = AccDev{0, 0, 0, 0, 0};
    ZShared ZS{nullptr, nullptr, nullptr};
    if (TRI) ZS = zshared_stage(VD, s_zt, s_zoff, s_z64, threadIdx.x, blockDim.x);
    __syncthreads();
    unsigned long long nmatch = 0;
    TriCtx C;
    if (TRI) tri_ctx_init(C, P, W);
    int cnt = 0;
    int prev_b = -1, ob = 0, hbits = 5, degb = 0;
    int64_t sb = 0;
    const int64_t mine = nunits > shard ? (nunits - shard + nshards - 1) / nshards : 0;
    for (;;) {
        unsigned long long jq = 0;
        if (lane == 0) jq = atomicAdd(queue, 1ull);
        jq = __shfl_sync(FULLMASK, jq, 0);
        if ((int64_t)jq >= mine) break;
        const int64_t tu = (int64_t)jq * nshards + shard;
        const uint64_t un = __ldg(units + tu);
        const int b = (int)(un >> 32), k = (int)(un & 0xffffffffu);
        if (b != prev_b) {                    // (re)build the table of N+(b)
            if (!TRI && prev_b >= 0) {
                __syncwarp();
                table_flush(O, sup, prev_b, ob, pay0, lane, 32);
            }
            const int64_t ob_ = __ldg(G.offs + b);
            sb = __ldg(O.split + b);
            ob = (int)(__ldg(G.offs + b + 1) - sb);
            degb = (int)(__ldg(G.offs + b + 1) - ob_);
            hbits = 5;
            while ((1 << hbits) < 2 * ob) ++hbits;
            __syncwarp();
            for (int i = lane; i < (1 << hbits); i += 32) key[i] = -1;
            __syncwarp();
            table_build<TRI>(G, O, sup, b, sb, ob, hbits, key, kpos, pay0, pay0, pay1, lane, 32);
            prev_b = b;
            __syncwarp();
        }
        if (TRI && W.degfilter && degb < C.mindeg1) continue;
        // the unit's FSGC_SUP_SEG in-entries in halves of kWSub (half the
        // slice arrays in shared memory per warp: more resident warps)
        const int64_t ibu = __ldg(G.offs + b) + (int64_t)k * FSGC_SUP_SEG;
        const int lenu = (int)min((int64_t)FSGC_SUP_SEG, sb - ibu);
        for (int h0 = 0; h0 < lenu; h0 += kWSub) {
            const int64_t ib0 = ibu + h0;
            const int len = min(kWSub, lenu - h0);
            const int64_t rbase = ib0 - __ldg(O.oofs + b);
            // slice setup: per in-entry a the start q0 of its tail (after b in
            // N+(a)) and the tail length; exclusive scan of the lengths -> pre
            int carry = 0;
            for (int j0 = 0; j0 < len; j0 += 32) {
                const int j = j0 + lane;
                int Lt = 0;
                if (j < len) {
                    const int a = __ldg(G.adj + ib0 + j);
                    const int e = __ldg(rev + rbase + j);
                    const int64_t sa = __ldg(O.split + a), oa = __ldg(O.oofs + a);
                    const int64_t q = sa + (e - oa) + 1;
                    Lt = (int)(__ldg(G.offs + a + 1) - q);
                    q0[j] = (uint32_t)q;
                    da[j] = (uint32_t)(sa - oa);
                    if (TRI) {
                        const int dga = (int)(__ldg(G.offs + a + 1) - __ldg(G.offs + a));
                        ea[j] = a;
                        xa[j] = dga;
                        ya[j] = __ldg(sup + e);
                        if (W.degfilter && dga < C.mindeg0) Lt = 0;
                        if (ya[j] == 0) Lt = 0;          // no triangle on (a, b)
                    } else {
                        ea[j] = e;
                        xa[j] = 0;
                    }
                }
                int x = Lt;                       // inclusive warp scan
    #pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int y = __shfl_up_sync(FULLMASK, x, o);
                    if (lane >= o) x += y;
                }
                if (j < len) pre[j] = carry + x - Lt;
                carry += __shfl_sync(FULLMASK, x, 31);
            }
            if (lane == 0) pre[len] = carry;
            __syncwarp();
            const int total = carry;
            int lo = 0;                           // monotone: last j with pre[j] <= idx
            for (int v0 = 0; v0 < total; v0 += 64) {
                int jj[2], cc[2];
                uint32_t pp[2];
                bool ok[2];
    #pragma unroll
                for (int r = 0; r < 2; ++r) {
                    const int idx = v0 + 32 * r + lane;
                    ok[r] = idx < total;
                    jj[r] = 0; pp[r] = 0; cc[r] = -1;
                    if (ok[r]) {
                        int l2 = lo, hi = len;
                        while (hi - l2 > 1) {
                            const int mid = (l2 + hi) >> 1;
                            if (pre[mid] <= idx) l2 = mid; else hi = mid;
                        }
                        lo = l2;
                        jj[r] = l2;
                        pp[r] = q0[l2] + (uint32_t)(idx - pre[l2]);
                        cc[r] = __ldg(G.adj + pp[r]);
                    }
                }
    #pragma unroll
                for (int r = 0; r < 2; ++r) {
                    const int h = ok[r] ? hfind(key, cc[r], hbits) : -1;
                    bool hit = h >= 0;
                    if (TRI) {
                        int dw = 0, cvw = 0;
                        if (hit) {
                            const int kk = kpos[h];
                            dw = pay1[kk];
                            cvw = pay0[kk];
                            if (W.degfilter && dw < C.mindeg2) hit = false;
                        }
                        cnt = tri_append(leaf, cnt, hit, ea[jj[r]], b, cc[r], xa[jj[r]], degb, dw, ya[jj[r]],
                                         pp[r] - da[jj[r]], cvw, lane);
                        if (cnt >= 32) {
                            tri_flush<NP, MODE == 2>(G, H, P, VD, C, sup, leaf, cnt, lrows, blockDim.x, wrows, lane, sa, ZS);
                            if (lane == 0) nmatch += cnt;
                            cnt = 0;
                        }
                    } else {
                        const unsigned hmask = __ballot_sync(FULLMASK, hit);
                        if (hit) {
                            atomicAdd(&pay0[kpos[h]], 1);                        // c(bc)
                            atomicAdd(sup + (pp[r] - da[jj[r]]), 1);             // c(ac)
                            const unsigned peers = __match_any_sync(hmask, jj[r]);   // c(ab): one add per a
                            if ((peers & ((1u << lane) - 1)) == 0) atomicAdd(&xa[jj[r]], __popc(peers));
                        }
                    }
                }
            }
            __syncwarp();
            if (!TRI) {
                for (int j = lane; j < len; j += 32)
                    if (xa[j]) atomicAdd(sup + ea[j], xa[j]);
            }
            __syncwarp();
        }
    }
    if (TRI) {
        if (cnt) {
            tri_flush<NP, MODE == 2>(G, H, P, VD, C, sup, leaf, cnt, lrows, blockDim.x, wrows, lane, sa, ZS);
            if (lane == 0) nmatch += cnt;
        }
        __shared__ unsigned long long s_nm[kWarpTabWarps];
        sacc_publish<NP>(s_acc, s_nm, kWarpTabWarps, nmatch, S, w, lane);
    } else if (prev_b >= 0) {
        __syncwarp();
        table_flush(O, sup, prev_b, ob, pay0, lane, 32);
    }
}

// ------------------------------------------------------------------------
// block-table kernel: the heavy middles.  Shared memory: the table of N+(b)
// (HS = pow2 >= 2 * max out(b) slots: key + payload), the block's unit and
// in-neighbour counters, per warp a leaf buffer and term rows (TRI).
// table bytes for hbits_max / max out(b): key + kpos per slot, then the
// payload per position in N+(b) (support: the c(b, x) counts; tri-core: tsup + tdeg)
__host__ __device__ inline size_t blocktab_table_bytes(int hs, int maxout, bool tri) {
    const size_t b = (size_t)hs * 6 + (size_t)maxout * (tri ? 8 : 4);
    return (b + 15) & ~(size_t)15;
}
__host__ __device__ inline size_t blocktab_warp_bytes(int mode) {   // leaf buffer (+ Venn warp rows, MODE 1)
    return mode ? (size_t)kLeafCap * kLeafW * 4 + (mode == 1 ? (size_t)kMaxVennRows * 16 : 0) : 0;
}

template <int MODE, int NP>
__global__ void __launch_bounds__((MODE == 1 ? kBlockTriWarps : MODE == 2 ? kBlockTriWarpsMax : kBlockTabWarps) * 32,
                                  MODE == 2 ? 2 : MODE)
    list_block_kernel(
    GraphDev G, OrientDev O, HubDev H, const int32_t* __restrict__ rev, const uint64_t* __restrict__ units,
    int64_t nunits, int hbits_max, int maxout, int* __restrict__ sup, unsigned long long* queue, int shard, int nshards,
    const __grid_constant__ CoreProg P, WorkDesc W, const __grid_constant__ VennDev VD, const Sink S) {
    constexpr bool TRI = MODE != 0;
    constexpr int NWBMAX = MODE == 1 ? kBlockTriWarps : MODE == 2 ? kBlockTriWarpsMax : kBlockTabWarps;
    const int NWB = blockDim.x >> 5;   // (MODE 2: the host's choice, <= NWBMAX)
    extern __shared__ __align__(16) unsigned char s_lb[];
    __shared__ long long s_unit;
    __shared__ int s_next;
    constexpr int kSubC = TRI ? kSubCTri : kSubCSup;
    __shared__ int32_t s_pre[kSubC + 1];          // sub-chunk: exclusive scan of the tail lengths
    __shared__ uint32_t s_q0[kSubC], s_da[kSubC];  // tail start in adj, split[a] - oofs[a]
    __shared__ int32_t s_e[kSubC], s_x[kSubC];     // support: e(ab), c(ab) count | tri-core: a, deg a
    __shared__ int32_t s_y[TRI ? kSubC : 1];       // tri-core: c(ab)
    __shared__ int32_t s_wsum[kSubC / 32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, tid = threadIdx.x, nthr = blockDim.x;
    const int HS = 1 << hbits_max;
    const size_t tab_b = blocktab_table_bytes(HS, maxout, TRI);
    int32_t* key = reinterpret_cast<int32_t*>(s_lb);
    int16_t* kpos = reinterpret_cast<int16_t*>(key + HS);
    int32_t* pay0 = reinterpret_cast<int32_t*>(kpos + HS);   // cnt[slot] | tsup[pos]
    int32_t* pay1 = pay0 + maxout;                            // - | tdeg[pos]
    unsigned char* wb = s_lb + tab_b + (size_t)w * blocktab_warp_bytes(MODE);
    uint32_t* leaf = reinterpret_cast<uint32_t*>(wb);
    u128* wrows = reinterpret_cast<u128*>(wb + (size_t)kLeafCap * kLeafW * 4);
    u128* lrows = reinterpret_cast<u128*>(s_lb + tab_b + NWB * blocktab_warp_bytes(MODE)) + tid;

    __shared__ AccDev s_acc[TRI ? NWBMAX : 1][TRI ? NP : 1];   // per-warp pattern sums (tri-core)
    __shared__ ZTerm s_zt[TRI ? kZShared : 1];
    __shared__ uint16_t s_zoff[FSGC_MAXPATS + 1];
    __shared__ int32_t s_z64[FSGC_MAXPATS];
    const SAcc sa{s_acc[TRI ? w : 0]};
    if (TRI && lane < NP) s_acc[w][lane] = AccDev{0, 0, 0, 0, 0};
    ZShared ZS{nullptr, nullptr, nullptr};
    if (TRI) ZS = zshared_stage(VD, s_zt, s_zoff, s_z64, tid, nthr);
    __syncthreads();
    unsigned long long nmatch = 0;
    TriCtx C;
    if (TRI) tri_ctx_init(C, P, W);
    int cnt = 0;
    int cur_b = -1, ob = 0, hbits = 5, degb = 0;
    int64_t sb = 0;
    const int64_t mine = nunits > shard ? (nunits - shard + nshards - 1) / nshards : 0;
    for (;;) {
        if (tid == 0) {
            const long long jq = (long long)atomicAdd(queue, 1ull);
            s_unit = jq < mine ? (long long)__ldg(units + (nunits - 1 - (jq * nshards + shard))) : -1ll;
            s_next = 0;
        }
        __syncthreads();
        const long long un = s_unit;
        if (un < 0) break;
        const int b = (int)((unsigned long long)un >> 32), k = (int)(un & 0xffffffffll);
        if (b != cur_b) {                      // (re)build the block's table of N+(b)
            if (!TRI && cur_b >= 0) table_flush(O, sup, cur_b, ob, pay0, tid, nthr);
            const int64_t ob_ = __ldg(G.offs + b);
            sb = __ldg(O.split + b);
            ob = (int)(__ldg(G.offs + b + 1) - sb);
            degb = (int)(__ldg(G.offs + b + 1) - ob_);
            hbits = 5;
            while ((1 << hbits) < 2 * ob) ++hbits;
            __syncthreads();
            for (int i = tid; i < (1 << hbits); i += nthr) key[i] = -1;
            __syncthreads();
            table_build<TRI>(G, O, sup, b, sb, ob, hbits, key, kpos, pay0, pay0, pay1, tid, nthr);
            cur_b = b;
            __syncthreads();
        }
        const bool skip = TRI && W.degfilter && degb < C.mindeg1;
        const int64_t ib0 = __ldg(G.offs + b) + (int64_t)k * FSGC_SUP_CHUNK;
        const int len = skip ? 0 : (int)min((int64_t)FSGC_SUP_CHUNK, sb - ib0);
        const int64_t rbase = ib0 - __ldg(O.oofs + b);
        // the unit in sub-chunks of kSubC in-entries; per sub-chunk the tails
        // are concatenated (block-wide exclusive scan of their lengths) and
        // the warps take 32 * kILP consecutive virtual elements at a time: the
        // work is balanced within the block whatever the tail lengths (the
        // heavy middles' tails are mostly short), and every lane has an
        // element each step
        for (int sc = 0; sc < len; sc += kSubC) {
            const int sl = min(kSubC, len - sc);
            for (int j = tid; j < kSubC; j += nthr) {
                int L = 0;
                if (j < sl) {
                    const int a = __ldg(G.adj + ib0 + sc + j);
                    const int e = __ldg(rev + rbase + sc + j);
                    const int64_t sa_ = __ldg(O.split + a), oa = __ldg(O.oofs + a);
                    const int64_t q = sa_ + (e - oa) + 1;
                    const int64_t ea = __ldg(G.offs + a + 1);
                    L = (int)(ea - q);
                    s_q0[j] = (uint32_t)q;
                    s_da[j] = (uint32_t)(sa_ - oa);
                    if (TRI) {
                        const int dga = (int)(ea - __ldg(G.offs + a));
                        const int cab = __ldg(sup + e);
                        s_e[j] = a;
                        s_x[j] = dga;
                        s_y[j] = cab;
                        if ((W.degfilter && dga < C.mindeg0) || cab == 0) L = 0;   // no triangle on (a, b)
                    } else {
                        s_e[j] = e;
                        s_x[j] = 0;
                    }
                }
                s_pre[j] = L;
            }
            if (tid == 0) s_next = 0;
            __syncthreads();
            {   // exclusive scan of s_pre[0, kSubC): 32-entry segments over the
                // warps (warp scans), then the segment offsets
                constexpr int NSEG = kSubC / 32;
                for (int sg = w; sg < NSEG; sg += NWB) {
                    const int j = sg * 32 + lane;
                    const int v = s_pre[j];
                    int x = v;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const int y = __shfl_up_sync(FULLMASK, x, o);
                        if (lane >= o) x += y;
                    }
                    s_pre[j] = x - v;
                    if (lane == 31) s_wsum[sg] = x;
                }
                __syncthreads();
                for (int sg = w; sg < NSEG; sg += NWB) {
                    int off = 0;
                    for (int q = 0; q < sg; ++q) off += s_wsum[q];
                    s_pre[sg * 32 + lane] += off;
                    if (sg == NSEG - 1 && lane == 31) s_pre[kSubC] = off + s_wsum[sg];
                }
                __syncthreads();
            }
            const int total = s_pre[kSubC];
            int lo = 0;                        // per lane: monotone over its elements
            for (;;) {
                int e0 = 0;
                if (lane == 0) e0 = atomicAdd(&s_next, 32 * kILP);
                e0 = __shfl_sync(FULLMASK, e0, 0);
                if (e0 >= total) break;
                int jj[kILP], cc[kILP];
                uint32_t pp[kILP];
#pragma unroll
                for (int r = 0; r < kILP; ++r) {   // last j with pre[j] <= idx: a non-empty tail
                    const int idx = e0 + 32 * r + lane;
                    jj[r] = 0; pp[r] = 0; cc[r] = -1;
                    if (idx < total) {
                        int l2 = lo;
                        if (s_pre[l2] > idx) l2 = 0;
                        // galloping from the lane's previous tail (the next
                        // element is usually in it or close), then bisection
                        int hi = l2 + 1, step = 1;
                        while (hi < kSubC && s_pre[hi] <= idx) {
                            l2 = hi;
                            step <<= 1;
                            hi = l2 + step;
                        }
                        if (hi > kSubC) hi = kSubC;
                        while (hi - l2 > 1) {
                            const int mid = (l2 + hi) >> 1;
                            if (s_pre[mid] <= idx) l2 = mid; else hi = mid;
                        }
                        lo = l2;
                        jj[r] = l2;
                        pp[r] = s_q0[l2] + (uint32_t)(idx - s_pre[l2]);
                        cc[r] = __ldg(G.adj + pp[r]);
                    }
                }
#pragma unroll
                for (int r = 0; r < kILP; ++r) {
                    const int h = cc[r] >= 0 ? hfind(key, cc[r], hbits) : -1;
                    bool hit = h >= 0;
                    const int j = jj[r];
                    if (TRI) {
                        int dw = 0, cvw = 0;
                        if (hit) {
                            const int kk = kpos[h];
                            dw = pay1[kk];
                            cvw = pay0[kk];
                            if (W.degfilter && dw < C.mindeg2) hit = false;
                        }
                        cnt = tri_append(leaf, cnt, hit, s_e[j], b, cc[r], s_x[j], degb, dw, s_y[j],
                                         pp[r] - s_da[j], cvw, lane);
                        if (cnt >= 32) {
                            tri_flush<NP, MODE == 2>(G, H, P, VD, C, sup, leaf, cnt, lrows, nthr, wrows, lane, sa, ZS);
                            if (lane == 0) nmatch += cnt;
                            cnt = 0;
                        }
                    } else {
                        const unsigned hmask = __ballot_sync(FULLMASK, hit);
                        if (hit) {
                            atomicAdd(&pay0[kpos[h]], 1);                  // c(bc)
                            atomicAdd(sup + (pp[r] - s_da[j]), 1);          // c(ac)
                            const unsigned peers = __match_any_sync(hmask, j);   // c(ab): one add per a
                            if ((peers & ((1u << lane) - 1)) == 0) atomicAdd(&s_x[j], __popc(peers));
                        }
                    }
                }
            }
            __syncthreads();
            if (!TRI) {
                for (int j = tid; j < sl; j += nthr)
                    if (s_x[j]) atomicAdd(sup + s_e[j], s_x[j]);
                __syncthreads();
            }
        }
        __syncthreads();
    }
    if (TRI) {
        if (cnt) {
            tri_flush<NP, MODE == 2>(G, H, P, VD, C, sup, leaf, cnt, lrows, nthr, wrows, lane, sa, ZS);
            if (lane == 0) nmatch += cnt;
        }
        __shared__ unsigned long long s_nm[NWBMAX];
        sacc_publish<NP>(s_acc, s_nm, NWB, nmatch, S, w, lane);
    } else if (cur_b >= 0) {
        table_flush(O, sup, cur_b, ob, pay0, tid, nthr);
    }
}
