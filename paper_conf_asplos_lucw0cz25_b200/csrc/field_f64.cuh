// field_f64.cuh -- BN254 Fr Montgomery products on the FP64 pipe (B200 runs DFMA at full rate:
// 63 DFMA/clk/SM measured, the same as IMAD), so products can be issued to a second, otherwise idle
// pipe next to the IMAD chains of field.cuh.
//
// Representation: radix W = 2^48, six limbs held as doubles (exact integers), R' = W^6 = 2^288.
// A limb product a*b (< 2^96, or |.| < 2^95 with a signed m) is split exactly with two FMAs:
//     t  = fma(a, b, C)         C = 1.5 * 2^100: the sum lies in [2^100, 2^101), ulp 2^48
//     hs = t - C                round(a*b / W) * W, exact
//     l  = fma(a, b, -hs)       a*b - hs in [-2^47, 2^47], exact
// l is added to column c and hs * 2^-48 to column c+1.  Column sums stay below 2^53 in magnitude
// (at most 18 terms of < 2^48 for two products plus the reduction), so every column is exact.
// CIOS row j: columns += x * y_j (+ u * v_j); m = (col_j mod W) * (-p^-1) mod W taken as a balanced
// residue in [-W/2, W/2]; columns += m * p (column j becomes a multiple of W); carry col_j / W.
// Result (columns 6..11) = (x y + u v + M p) / 2^288 lies in (-p/2 - e, p/2 + e) for inputs < 2^256,
// so one conditional addition of p makes it canonical.
#pragma once
#include <stdint.h>
#include "field.cuh"

namespace bzk {

struct f6 { double d[6]; };

#define BZK_F_C 0x1.8p+100                /* 1.5 * 2^100 (exact hex-float literals throughout) */
#define BZK_F_C2 0x1.8p+52                /* 1.5 * 2^52  */
#define BZK_F_W 0x1p+48                   /* 2^48        */
#define BZK_F_IW 0x1p-48                  /* 2^-48       */

// p in radix 2^48 and -p^{-1} mod 2^48
__device__ __forceinline__ double fp_limb(int i) {
    switch (i) {
        case 0: return (double)0xf593f0000001ull;
        case 1: return (double)0x79b9709143e1ull;
        case 2: return (double)0x585d2833e848ull;
        case 3: return (double)0xb85045b68181ull;
        case 4: return (double)0x4e72e131a029ull;
        default: return (double)0x3064ull;
    }
}
#define BZK_F_NP ((double)0xf593efffffffull)   /* -p^{-1} mod 2^48 */

// 48-bit unsigned integer (< 2^48) -> exact double (magic exponent 2^52)
__device__ __forceinline__ double u48_to_f(uint32_t lo, uint32_t hi16) {
    return __hiloint2double((int)(0x43300000u | hi16), (int)lo) - 0x1p+52;
}

// 256-bit integer (8 x u32, any value < 2^256) -> six 48-bit limbs
__device__ __forceinline__ f6 to_f6(const fe &x) {
    f6 r;
    r.d[0] = u48_to_f(x.l[0], x.l[1] & 0xffffu);
    r.d[1] = u48_to_f(__funnelshift_r(x.l[1], x.l[2], 16), x.l[2] >> 16);
    r.d[2] = u48_to_f(x.l[3], x.l[4] & 0xffffu);
    r.d[3] = u48_to_f(__funnelshift_r(x.l[4], x.l[5], 16), x.l[5] >> 16);
    r.d[4] = u48_to_f(x.l[6], x.l[7] & 0xffffu);
    r.d[5] = u48_to_f(x.l[7] >> 16, 0u);
    return r;
}

// accumulate a * b into columns c, c+1
__device__ __forceinline__ void f_mac(double a, double b, double &lo, double &hi) {
    const double t = __fma_rn(a, b, BZK_F_C);
    const double hs = t - BZK_F_C;
    lo += __fma_rn(a, b, -hs);
    hi = __fma_rn(hs, BZK_F_IW, hi);
}

// (x*y [+ u*v]) * 2^-288 mod p, canonical.  NP = 1 or 2 products.
template <int NP>
__device__ __forceinline__ fe fmont(const f6 &x, const f6 &y, const f6 &u, const f6 &v) {
    double col[13];
#pragma unroll
    for (int c = 0; c < 13; ++c) col[c] = 0.0;
#pragma unroll
    for (int j = 0; j < 6; ++j) {
#pragma unroll
        for (int i = 0; i < 6; ++i) {
            f_mac(x.d[i], y.d[j], col[i + j], col[i + j + 1]);
            if (NP == 2) f_mac(u.d[i], v.d[j], col[i + j], col[i + j + 1]);
        }
        // balanced residue of column j, then m = u * (-p^-1) mod W (balanced)
        const double q = __fma_rn(col[j], BZK_F_IW, BZK_F_C2) - BZK_F_C2;
        const double uj = __fma_rn(q, -BZK_F_W, col[j]);
        const double t = __fma_rn(uj, BZK_F_NP, BZK_F_C);
        const double hs = t - BZK_F_C;
        const double m = __fma_rn(uj, BZK_F_NP, -hs);
#pragma unroll
        for (int i = 0; i < 6; ++i) f_mac(m, fp_limb(i), col[j + i], col[j + i + 1]);
        col[j + 1] = __fma_rn(col[j], BZK_F_IW, col[j + 1]);   // col[j] is now a multiple of W
    }
    // columns 6..11 -> digits in [0, W) (floor division), sign in column 12 (0 or -1)
    uint32_t lo[6], hi[6];
#pragma unroll
    for (int c = 6; c < 12; ++c) {
        const double q = __fma_rd(col[c], BZK_F_IW, BZK_F_C2) - BZK_F_C2;   // floor(col / W)
        const double r = __fma_rn(q, -BZK_F_W, col[c]);                     // in [0, W), exact
        col[c + 1] += q;
        const double rb = r + 0x1p+52;                          // bits: 2^52 | r
        lo[c - 6] = (uint32_t)__double2loint(rb);
        hi[c - 6] = (uint32_t)__double2hiint(rb) & 0xffffu;
    }
    // low 256 bits of sum_k digit_k 2^(48k)
    fe r;
    r.l[0] = lo[0];
    r.l[1] = hi[0] | (lo[1] << 16);
    r.l[2] = __funnelshift_r(lo[1], hi[1], 16);
    r.l[3] = lo[2];
    r.l[4] = hi[2] | (lo[3] << 16);
    r.l[5] = __funnelshift_r(lo[3], hi[3], 16);
    r.l[6] = lo[4];
    r.l[7] = hi[4] | (lo[5] << 16);
    const uint32_t neg = col[12] < 0.0 ? 0xffffffffu : 0u;
    // negative result: add p (T + p < p; the addition mod 2^256 gives it exactly)
    fe pm;
    pm.l[0] = BZK_P0 & neg; pm.l[1] = BZK_P1 & neg; pm.l[2] = BZK_P2 & neg; pm.l[3] = BZK_P3 & neg;
    pm.l[4] = BZK_P4 & neg; pm.l[5] = BZK_P5 & neg; pm.l[6] = BZK_P6 & neg; pm.l[7] = BZK_P7 & neg;
    return lz_add(r, pm);
}

}  // namespace bzk
