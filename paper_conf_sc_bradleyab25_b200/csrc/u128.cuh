// u128.cuh -- exact unsigned 128-bit arithmetic with overflow detection,
// usable on host and device (north_star: "exact unsigned 128-bit count").
// Every operation returns the wrapped result and ORs an overflow flag so a
// count that does not fit 2^128 - 1 is reported, never silently wrapped.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define FSGC_HD __host__ __device__ __forceinline__
#else
#define FSGC_HD inline
#endif

typedef unsigned __int128 u128;

FSGC_HD uint64_t u128_lo(u128 x) { return (uint64_t)x; }
FSGC_HD uint64_t u128_hi(u128 x) { return (uint64_t)(x >> 64); }
FSGC_HD u128 u128_make(uint64_t lo, uint64_t hi) { return ((u128)hi << 64) | lo; }

FSGC_HD u128 add_ovf(u128 a, u128 b, bool& ovf) {
    u128 r = a + b;
    ovf |= (r < a);
    return r;
}

FSGC_HD uint64_t mulhi64(uint64_t a, uint64_t b) {
#ifdef __CUDA_ARCH__
    return __umul64hi(a, b);
#else
    return (uint64_t)(((u128)a * b) >> 64);
#endif
}

// a * b (128 x 64), overflow if the product needs more than 128 bits
FSGC_HD u128 mul_ovf64(u128 a, uint64_t b, bool& ovf) {
    uint64_t alo = u128_lo(a), ahi = u128_hi(a);
    u128 lo = (u128)alo * b;                 // <= 128 bits
    uint64_t hhi = mulhi64(ahi, b);          // bits 128..191 of ahi*b*2^64
    uint64_t hlo = ahi * b;                  // bits 64..127
    ovf |= (hhi != 0);
    u128 r = lo + ((u128)hlo << 64);
    ovf |= (u128_hi(r) < hlo);               // carry out of bit 127
    return r;
}

// a * b (128 x 128)
FSGC_HD u128 mul_ovf(u128 a, u128 b, bool& ovf) {
    if (u128_hi(a) != 0 && u128_hi(b) != 0) {
        ovf = true;
        return a * b;
    }
    if (u128_hi(b) == 0) return mul_ovf64(a, u128_lo(b), ovf);
    return mul_ovf64(b, u128_lo(a), ovf);
}

// binom(n, k) for n < 2^63, k <= 64: r_i = r_{i-1} * (n-k+i) / i is exact at
// every step (r_i = C(n-k+i, i)); the 192-bit intermediate r * (n-k+i) is
// divided by i with 32-bit limbs, so the result is exact whenever it fits.
FSGC_HD u128 binom_ovf(uint64_t n, uint32_t k, bool& ovf) {
    if (k > n) return 0;
    if (k == 0) return 1;
    if (k == 1) return n;
    if (k == 2) {
        uint64_t a = n, b = n - 1;
        if (a & 1) b >>= 1; else a >>= 1;
        return (u128)a * b;
    }
    u128 r = 1;
    for (uint32_t i = 1; i <= k; ++i) {
        uint64_t f = n - k + i;
        // 192-bit product p = r * f as (p2 : p1 : p0) 64-bit words
        uint64_t r0 = u128_lo(r), r1 = u128_hi(r);
        u128 t0 = (u128)r0 * f;
        u128 t1 = (u128)r1 * f + (uint64_t)(t0 >> 64);
        uint64_t p0 = (uint64_t)t0, p1 = (uint64_t)t1, p2 = (uint64_t)(t1 >> 64);
        // divide by i (32 bit) limb by limb, most significant first
        uint32_t limb[6] = {(uint32_t)(p2 >> 32), (uint32_t)p2, (uint32_t)(p1 >> 32),
                            (uint32_t)p1, (uint32_t)(p0 >> 32), (uint32_t)p0};
        uint64_t rem = 0;
        uint32_t q[6];
#pragma unroll
        for (int j = 0; j < 6; ++j) {
            uint64_t cur = (rem << 32) | limb[j];
            q[j] = (uint32_t)(cur / i);
            rem = cur % i;
        }
        if (q[0] | q[1]) { ovf = true; }
        r = u128_make(((uint64_t)q[4] << 32) | q[5], ((uint64_t)q[2] << 32) | q[3]);
    }
    return r;
}
