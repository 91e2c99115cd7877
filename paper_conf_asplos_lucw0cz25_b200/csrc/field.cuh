// field.cuh -- BN254 scalar field F_p on sm_100a: 8 x 32-bit limbs, Montgomery CIOS on
// 32-bit IMAD carry chains (mad.lo.cc / madc.hi.cc).
//
// Reading R1: the paper fixes 256-bit elements (PAPER.md:187 Sec. 3.3, :320
// Sec. 6.2) but never names the prime; we take BN254 Fr.
//
// Representation conventions used by the kernels:
//   * tables and every value that leaves the library are in STANDARD form, canonical (< p);
//   * challenges are held in MONTGOMERY form (r*R mod p, R = 2^256) so that
//     mont_mul(r*R, x) = r*x: the fold T' = a + r(b - a) stays in standard form with ONE
//     mont_mul and no conversion pass;
//   * a product of d standard values through d-1 mont_muls carries R^{-(d-1)}; round sums
//     are fixed once per round by mont_mul(S, R^d mod p).
#pragma once
#include <stdint.h>

namespace bzk {

struct fe { uint32_t l[8]; };

// p = 0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001 (LE 32-bit limbs)
#define BZK_P0 0xf0000001u
#define BZK_P1 0x43e1f593u
#define BZK_P2 0x79b97091u
#define BZK_P3 0x2833e848u
#define BZK_P4 0x8181585du
#define BZK_P5 0xb85045b6u
#define BZK_P6 0xe131a029u
#define BZK_P7 0x30644e72u
#define BZK_NP0 0xefffffffu   // -p^{-1} mod 2^32

// Constants in standard form (LE limbs), derived in DESIGN.md App. A and checked on the host
// by tests/test_abi.py against Python integers (bzk_debug_constants).
//   R mod p, R^2 mod p, R^3 mod p, R^4 mod p, R^5 mod p
__device__ __forceinline__ fe fe_const(int which);

__device__ __forceinline__ fe fe_zero() { fe r; _Pragma("unroll") for (int i = 0; i < 8; ++i) r.l[i] = 0; return r; }

__device__ __forceinline__ bool fe_is_zero(const fe &a) {
    uint32_t x = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) x |= a.l[i];
    return x == 0;
}

// r = a - p (with borrow out); returns borrow (1 if a < p)
__device__ __forceinline__ uint32_t sub_p(fe &r, const fe &a) {
    uint32_t borrow;
    asm("sub.cc.u32  %0, %9,  %17;\n\t"
        "subc.cc.u32 %1, %10, %18;\n\t"
        "subc.cc.u32 %2, %11, %19;\n\t"
        "subc.cc.u32 %3, %12, %20;\n\t"
        "subc.cc.u32 %4, %13, %21;\n\t"
        "subc.cc.u32 %5, %14, %22;\n\t"
        "subc.cc.u32 %6, %15, %23;\n\t"
        "subc.cc.u32 %7, %16, %24;\n\t"
        "subc.u32    %8, 0, 0;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]),
          "=r"(r.l[6]), "=r"(r.l[7]), "=r"(borrow)
        : "r"(a.l[0]), "r"(a.l[1]), "r"(a.l[2]), "r"(a.l[3]), "r"(a.l[4]), "r"(a.l[5]), "r"(a.l[6]),
          "r"(a.l[7]), "n"(BZK_P0), "n"(BZK_P1), "n"(BZK_P2), "n"(BZK_P3), "n"(BZK_P4), "n"(BZK_P5),
          "n"(BZK_P6), "n"(BZK_P7));
    return borrow;   // 0xffffffff if a < p, else 0
}

// a mod p for a < 2p
__device__ __forceinline__ fe fe_reduce_once(const fe &a) {
    fe s;
    uint32_t borrow = sub_p(s, a);
    fe r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.l[i] = borrow ? a.l[i] : s.l[i];
    return r;
}

// (a + b) mod p for canonical a, b (a + b < 2p < 2^255: no carry out of 256 bits)
__device__ __forceinline__ fe fe_add(const fe &a, const fe &b) {
    fe s;
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(s.l[0]), "=r"(s.l[1]), "=r"(s.l[2]), "=r"(s.l[3]), "=r"(s.l[4]), "=r"(s.l[5]),
          "=r"(s.l[6]), "=r"(s.l[7])
        : "r"(a.l[0]), "r"(a.l[1]), "r"(a.l[2]), "r"(a.l[3]), "r"(a.l[4]), "r"(a.l[5]), "r"(a.l[6]),
          "r"(a.l[7]), "r"(b.l[0]), "r"(b.l[1]), "r"(b.l[2]), "r"(b.l[3]), "r"(b.l[4]), "r"(b.l[5]),
          "r"(b.l[6]), "r"(b.l[7]));
    return fe_reduce_once(s);
}

// (a - b) mod p for canonical a, b
__device__ __forceinline__ fe fe_sub(const fe &a, const fe &b) {
    fe s;
    uint32_t borrow;
    asm("sub.cc.u32  %0, %9,  %17;\n\t"
        "subc.cc.u32 %1, %10, %18;\n\t"
        "subc.cc.u32 %2, %11, %19;\n\t"
        "subc.cc.u32 %3, %12, %20;\n\t"
        "subc.cc.u32 %4, %13, %21;\n\t"
        "subc.cc.u32 %5, %14, %22;\n\t"
        "subc.cc.u32 %6, %15, %23;\n\t"
        "subc.cc.u32 %7, %16, %24;\n\t"
        "subc.u32    %8, 0, 0;"
        : "=r"(s.l[0]), "=r"(s.l[1]), "=r"(s.l[2]), "=r"(s.l[3]), "=r"(s.l[4]), "=r"(s.l[5]),
          "=r"(s.l[6]), "=r"(s.l[7]), "=r"(borrow)
        : "r"(a.l[0]), "r"(a.l[1]), "r"(a.l[2]), "r"(a.l[3]), "r"(a.l[4]), "r"(a.l[5]), "r"(a.l[6]),
          "r"(a.l[7]), "r"(b.l[0]), "r"(b.l[1]), "r"(b.l[2]), "r"(b.l[3]), "r"(b.l[4]), "r"(b.l[5]),
          "r"(b.l[6]), "r"(b.l[7]));
    // add back p masked by the borrow
    uint32_t m0 = BZK_P0 & borrow, m1 = BZK_P1 & borrow, m2 = BZK_P2 & borrow, m3 = BZK_P3 & borrow;
    uint32_t m4 = BZK_P4 & borrow, m5 = BZK_P5 & borrow, m6 = BZK_P6 & borrow, m7 = BZK_P7 & borrow;
    asm("add.cc.u32  %0, %0, %8;\n\t"
        "addc.cc.u32 %1, %1, %9;\n\t"
        "addc.cc.u32 %2, %2, %10;\n\t"
        "addc.cc.u32 %3, %3, %11;\n\t"
        "addc.cc.u32 %4, %4, %12;\n\t"
        "addc.cc.u32 %5, %5, %13;\n\t"
        "addc.cc.u32 %6, %6, %14;\n\t"
        "addc.u32    %7, %7, %15;"
        : "+r"(s.l[0]), "+r"(s.l[1]), "+r"(s.l[2]), "+r"(s.l[3]), "+r"(s.l[4]), "+r"(s.l[5]),
          "+r"(s.l[6]), "+r"(s.l[7])
        : "r"(m0), "r"(m1), "r"(m2), "r"(m3), "r"(m4), "r"(m5), "r"(m6), "r"(m7));
    return s;
}

// t[0..9] += a[0..7] * b   (even-index products on one carry chain, odd on another)
__device__ __forceinline__ void mad_row(uint32_t t[10], const uint32_t a[8], uint32_t b) {
    asm("mad.lo.cc.u32  %0, %10, %18, %0;\n\t"
        "madc.hi.cc.u32 %1, %10, %18, %1;\n\t"
        "madc.lo.cc.u32 %2, %12, %18, %2;\n\t"
        "madc.hi.cc.u32 %3, %12, %18, %3;\n\t"
        "madc.lo.cc.u32 %4, %14, %18, %4;\n\t"
        "madc.hi.cc.u32 %5, %14, %18, %5;\n\t"
        "madc.lo.cc.u32 %6, %16, %18, %6;\n\t"
        "madc.hi.cc.u32 %7, %16, %18, %7;\n\t"
        "addc.cc.u32    %8, %8, 0;\n\t"
        "addc.u32       %9, %9, 0;\n\t"
        "mad.lo.cc.u32  %1, %11, %18, %1;\n\t"
        "madc.hi.cc.u32 %2, %11, %18, %2;\n\t"
        "madc.lo.cc.u32 %3, %13, %18, %3;\n\t"
        "madc.hi.cc.u32 %4, %13, %18, %4;\n\t"
        "madc.lo.cc.u32 %5, %15, %18, %5;\n\t"
        "madc.hi.cc.u32 %6, %15, %18, %6;\n\t"
        "madc.lo.cc.u32 %7, %17, %18, %7;\n\t"
        "madc.hi.cc.u32 %8, %17, %18, %8;\n\t"
        "addc.u32       %9, %9, 0;"
        : "+r"(t[0]), "+r"(t[1]), "+r"(t[2]), "+r"(t[3]), "+r"(t[4]), "+r"(t[5]), "+r"(t[6]),
          "+r"(t[7]), "+r"(t[8]), "+r"(t[9])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(a[4]), "r"(a[5]), "r"(a[6]), "r"(a[7]),
          "r"(b));
}

// t[0..9] += p * m
__device__ __forceinline__ void mad_row_p(uint32_t t[10], uint32_t m) {
    asm("mad.lo.cc.u32  %0, %11, %10, %0;\n\t"
        "madc.hi.cc.u32 %1, %11, %10, %1;\n\t"
        "madc.lo.cc.u32 %2, %13, %10, %2;\n\t"
        "madc.hi.cc.u32 %3, %13, %10, %3;\n\t"
        "madc.lo.cc.u32 %4, %15, %10, %4;\n\t"
        "madc.hi.cc.u32 %5, %15, %10, %5;\n\t"
        "madc.lo.cc.u32 %6, %17, %10, %6;\n\t"
        "madc.hi.cc.u32 %7, %17, %10, %7;\n\t"
        "addc.cc.u32    %8, %8, 0;\n\t"
        "addc.u32       %9, %9, 0;\n\t"
        "mad.lo.cc.u32  %1, %12, %10, %1;\n\t"
        "madc.hi.cc.u32 %2, %12, %10, %2;\n\t"
        "madc.lo.cc.u32 %3, %14, %10, %3;\n\t"
        "madc.hi.cc.u32 %4, %14, %10, %4;\n\t"
        "madc.lo.cc.u32 %5, %16, %10, %5;\n\t"
        "madc.hi.cc.u32 %6, %16, %10, %6;\n\t"
        "madc.lo.cc.u32 %7, %18, %10, %7;\n\t"
        "madc.hi.cc.u32 %8, %18, %10, %8;\n\t"
        "addc.u32       %9, %9, 0;"
        : "+r"(t[0]), "+r"(t[1]), "+r"(t[2]), "+r"(t[3]), "+r"(t[4]), "+r"(t[5]), "+r"(t[6]),
          "+r"(t[7]), "+r"(t[8]), "+r"(t[9])
        : "r"(m), "r"(BZK_P0), "r"(BZK_P1), "r"(BZK_P2), "r"(BZK_P3), "r"(BZK_P4), "r"(BZK_P5),
          "r"(BZK_P6), "r"(BZK_P7));
}

// Montgomery product a*b*R^{-1} mod p (CIOS, row-wise), reference version kept for the
// micro-benchmark (bzk_debug_bench kind 2): a single 10-word accumulator, even/odd product chains.
__device__ __forceinline__ fe mont_mul_v1(const fe &a, const fe &b) {
    uint32_t t[10];
#pragma unroll
    for (int i = 0; i < 10; ++i) t[i] = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        mad_row(t, a.l, b.l[i]);
        uint32_t m = t[0] * BZK_NP0;
        mad_row_p(t, m);
#pragma unroll
        for (int j = 0; j < 9; ++j) t[j] = t[j + 1];
        t[9] = 0;
    }
    fe r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.l[i] = t[i];
    return fe_reduce_once(r);
}

// ---------------------------------------------------------------- Montgomery product (hot path)
//
// CIOS with two parity-aligned accumulators so that every 32x32->64 product lands in an aligned
// register pair and ptxas can emit one IMAD.WIDE.U32(.X) per product with no register moves:
//   A[q] holds relative column q (pairs (A0,A1),(A2,A3),...,(A6,A7), A8 single),
//   B[q] holds relative column q+1 (pairs (B0,B1) at columns (1,2), ..., B8 at column 9),
//   L    holds a pending word at column 0.
// Row i: A += a_even * b_i, B += a_odd * b_i (L is folded in at the head of the B chain, whose
// carry enters column 1 = B0), m = A0 * (-p^{-1}), A += p_even * m, B += p_odd * m, then divide by
// W = 2^32: the new A is the old B (columns 1..9), the new B is old A2..A8, and old A1 (column 1)
// becomes the new pending L.  After 8 rows: result = A + L + (B << 32).

// B chain of a row: A0 += L (carry to column 1), B[0..7] += a_odd * bi, carry into B8
__device__ __forceinline__ void row_b(uint32_t A[9], uint32_t B[9], uint32_t L, const uint32_t a[8], uint32_t bi) {
    asm("add.cc.u32     %0, %0, %10;\n\t"
        "madc.lo.cc.u32 %1, %11, %15, %1;\n\t"
        "madc.hi.cc.u32 %2, %11, %15, %2;\n\t"
        "madc.lo.cc.u32 %3, %12, %15, %3;\n\t"
        "madc.hi.cc.u32 %4, %12, %15, %4;\n\t"
        "madc.lo.cc.u32 %5, %13, %15, %5;\n\t"
        "madc.hi.cc.u32 %6, %13, %15, %6;\n\t"
        "madc.lo.cc.u32 %7, %14, %15, %7;\n\t"
        "madc.hi.cc.u32 %8, %14, %15, %8;\n\t"
        "addc.u32       %9, %9, 0;"
        : "+r"(A[0]), "+r"(B[0]), "+r"(B[1]), "+r"(B[2]), "+r"(B[3]), "+r"(B[4]), "+r"(B[5]), "+r"(B[6]),
          "+r"(B[7]), "+r"(B[8])
        : "r"(L), "r"(a[1]), "r"(a[3]), "r"(a[5]), "r"(a[7]), "r"(bi));
}

// Same as row_b when B7 == B8 == 0 on entry (the first B chain of a row after the shift): the top
// product is written, not accumulated, and no zero needs to be materialised (no IMAD.MOV).
__device__ __forceinline__ void row_b_z(uint32_t A[9], uint32_t B[9], uint32_t L, const uint32_t a[8], uint32_t bi) {
    asm("add.cc.u32     %0, %0, %10;\n\t"
        "madc.lo.cc.u32 %1, %11, %15, %1;\n\t"
        "madc.hi.cc.u32 %2, %11, %15, %2;\n\t"
        "madc.lo.cc.u32 %3, %12, %15, %3;\n\t"
        "madc.hi.cc.u32 %4, %12, %15, %4;\n\t"
        "madc.lo.cc.u32 %5, %13, %15, %5;\n\t"
        "madc.hi.cc.u32 %6, %13, %15, %6;\n\t"
        "madc.lo.cc.u32 %7, %14, %15, %7;\n\t"
        "madc.hi.cc.u32 %8, %14, %15, 0;\n\t"
        "addc.u32       %9, 0, 0;"
        : "+r"(A[0]), "+r"(B[0]), "+r"(B[1]), "+r"(B[2]), "+r"(B[3]), "+r"(B[4]), "+r"(B[5]), "+r"(B[6]),
          "=r"(B[7]), "=r"(B[8])
        : "r"(L), "r"(a[1]), "r"(a[3]), "r"(a[5]), "r"(a[7]), "r"(bi));
}

// B chain without a pending word: B[0..7] += a_odd * bi, carry into B8 (second product of a row)
__device__ __forceinline__ void row_b_nl(uint32_t B[9], const uint32_t a[8], uint32_t bi) {
    asm("mad.lo.cc.u32  %0, %9,  %13, %0;\n\t"
        "madc.hi.cc.u32 %1, %9,  %13, %1;\n\t"
        "madc.lo.cc.u32 %2, %10, %13, %2;\n\t"
        "madc.hi.cc.u32 %3, %10, %13, %3;\n\t"
        "madc.lo.cc.u32 %4, %11, %13, %4;\n\t"
        "madc.hi.cc.u32 %5, %11, %13, %5;\n\t"
        "madc.lo.cc.u32 %6, %12, %13, %6;\n\t"
        "madc.hi.cc.u32 %7, %12, %13, %7;\n\t"
        "addc.u32       %8, %8, 0;"
        : "+r"(B[0]), "+r"(B[1]), "+r"(B[2]), "+r"(B[3]), "+r"(B[4]), "+r"(B[5]), "+r"(B[6]), "+r"(B[7]),
          "+r"(B[8])
        : "r"(a[1]), "r"(a[3]), "r"(a[5]), "r"(a[7]), "r"(bi));
}

// A chain of a row: A[0..7] += a_even * bi, carry into A8
__device__ __forceinline__ void row_a(uint32_t A[9], const uint32_t a[8], uint32_t bi) {
    asm("mad.lo.cc.u32  %0, %9,  %13, %0;\n\t"
        "madc.hi.cc.u32 %1, %9,  %13, %1;\n\t"
        "madc.lo.cc.u32 %2, %10, %13, %2;\n\t"
        "madc.hi.cc.u32 %3, %10, %13, %3;\n\t"
        "madc.lo.cc.u32 %4, %11, %13, %4;\n\t"
        "madc.hi.cc.u32 %5, %11, %13, %5;\n\t"
        "madc.lo.cc.u32 %6, %12, %13, %6;\n\t"
        "madc.hi.cc.u32 %7, %12, %13, %7;\n\t"
        "addc.u32       %8, %8, 0;"
        : "+r"(A[0]), "+r"(A[1]), "+r"(A[2]), "+r"(A[3]), "+r"(A[4]), "+r"(A[5]), "+r"(A[6]), "+r"(A[7]),
          "+r"(A[8])
        : "r"(a[0]), "r"(a[2]), "r"(a[4]), "r"(a[6]), "r"(bi));
}

// reduction chains: A += p_even * m (A0 -> 0), B += p_odd * m, m = A0 * (-p^{-1}) mod 2^32
__device__ __forceinline__ uint32_t mont_m(uint32_t a0) { return a0 * BZK_NP0; }

__device__ __forceinline__ void red_a(uint32_t A[9], uint32_t m) {
    asm("mad.lo.cc.u32  %0, %9, %10, %0;\n\t"
        "madc.hi.cc.u32 %1, %9, %10, %1;\n\t"
        "madc.lo.cc.u32 %2, %9, %11, %2;\n\t"
        "madc.hi.cc.u32 %3, %9, %11, %3;\n\t"
        "madc.lo.cc.u32 %4, %9, %12, %4;\n\t"
        "madc.hi.cc.u32 %5, %9, %12, %5;\n\t"
        "madc.lo.cc.u32 %6, %9, %13, %6;\n\t"
        "madc.hi.cc.u32 %7, %9, %13, %7;\n\t"
        "addc.u32       %8, %8, 0;"
        : "+r"(A[0]), "+r"(A[1]), "+r"(A[2]), "+r"(A[3]), "+r"(A[4]), "+r"(A[5]), "+r"(A[6]), "+r"(A[7]),
          "+r"(A[8])
        : "r"(m), "n"(BZK_P0), "n"(BZK_P2), "n"(BZK_P4), "n"(BZK_P6));
}

__device__ __forceinline__ void red_b(uint32_t B[9], uint32_t m) {
    asm("mad.lo.cc.u32  %0, %9, %10, %0;\n\t"
        "madc.hi.cc.u32 %1, %9, %10, %1;\n\t"
        "madc.lo.cc.u32 %2, %9, %11, %2;\n\t"
        "madc.hi.cc.u32 %3, %9, %11, %3;\n\t"
        "madc.lo.cc.u32 %4, %9, %12, %4;\n\t"
        "madc.hi.cc.u32 %5, %9, %12, %5;\n\t"
        "madc.lo.cc.u32 %6, %9, %13, %6;\n\t"
        "madc.hi.cc.u32 %7, %9, %13, %7;\n\t"
        "addc.u32       %8, %8, 0;"
        : "+r"(B[0]), "+r"(B[1]), "+r"(B[2]), "+r"(B[3]), "+r"(B[4]), "+r"(B[5]), "+r"(B[6]), "+r"(B[7]),
          "+r"(B[8])
        : "r"(m), "n"(BZK_P1), "n"(BZK_P3), "n"(BZK_P5), "n"(BZK_P7));
}

// Lazy Montgomery product: returns t = a*b*R^{-1} + q*p < a*b/R + p (no final subtraction).
// With p/R = 0.189 (BN254): a, b < 2p, or a < 4p and b < p  ->  t < 1.76p.
__device__ __forceinline__ fe mont_mul_lz(const fe &a, const fe &b) {
    uint32_t A[9], B[9], L = 0;
    // row 0: plain products (no accumulation)
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(A[0]), "=r"(A[1]), "=r"(A[2]), "=r"(A[3]), "=r"(A[4]), "=r"(A[5]), "=r"(A[6]), "=r"(A[7]),
          "=r"(A[8])
        : "r"(a.l[0]), "r"(a.l[2]), "r"(a.l[4]), "r"(a.l[6]), "r"(b.l[0]));
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(B[0]), "=r"(B[1]), "=r"(B[2]), "=r"(B[3]), "=r"(B[4]), "=r"(B[5]), "=r"(B[6]), "=r"(B[7]),
          "=r"(B[8])
        : "r"(a.l[1]), "r"(a.l[3]), "r"(a.l[5]), "r"(a.l[7]), "r"(b.l[0]));
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        if (i > 0) {
            row_b_z(A, B, L, a.l, b.l[i]);
            row_a(A, a.l, b.l[i]);
        }
        uint32_t m = mont_m(A[0]);
        red_a(A, m);
        red_b(B, m);
        // divide by W: L = A1; A <- B; B <- A2..A8, 0, 0
        L = A[1];
        uint32_t nA[9], nB[9];
#pragma unroll
        for (int q = 0; q < 9; ++q) nA[q] = B[q];
#pragma unroll
        for (int q = 0; q < 7; ++q) nB[q] = A[q + 2];
        nB[7] = 0;
        nB[8] = 0;
#pragma unroll
        for (int q = 0; q < 9; ++q) { A[q] = nA[q]; B[q] = nB[q]; }
    }
    // result = A + L + (B << 32)   (< 2p < 2^255, so A8 and B7, B8 end up zero)
    fe r;
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]), "=r"(r.l[6]),
          "=r"(r.l[7])
        : "r"(A[0]), "r"(A[1]), "r"(A[2]), "r"(A[3]), "r"(A[4]), "r"(A[5]), "r"(A[6]), "r"(A[7]),
          "r"(L), "r"(B[0]), "r"(B[1]), "r"(B[2]), "r"(B[3]), "r"(B[4]), "r"(B[5]), "r"(B[6]));
    return r;
}

// Montgomery product a*b*R^{-1} mod p; a, b canonical -> canonical.
__device__ __forceinline__ fe mont_mul(const fe &a, const fe &b) { return fe_reduce_once(mont_mul_lz(a, b)); }

// The same product, NOT inlined: for the one-thread-per-proof serial work of a round (finalisation,
// Lagrange), where one shared copy of the code stays in the instruction cache across call sites.
static __device__ __noinline__ fe mont_mul_serial(const fe a, const fe b) { return mont_mul(a, b); }

// (x*y + u*v) * R^{-1} (+ q p) with ONE Montgomery reduction (lazy sum of two products).
// Each row adds x*y_i and u*v_i before the reduction row.  Result < (x*y + u*v)/R + p: with
// x, y, u, v < 2p it is < 2.52p (< 2^256 since 4p < 2^256); with x, u < p, y, v < 2^256 it is < 3p.
__device__ __forceinline__ fe mont_mul2_lz(const fe &x, const fe &y, const fe &u, const fe &v) {
    uint32_t A[9], B[9], L = 0;
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(A[0]), "=r"(A[1]), "=r"(A[2]), "=r"(A[3]), "=r"(A[4]), "=r"(A[5]), "=r"(A[6]), "=r"(A[7]),
          "=r"(A[8])
        : "r"(x.l[0]), "r"(x.l[2]), "r"(x.l[4]), "r"(x.l[6]), "r"(y.l[0]));
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(B[0]), "=r"(B[1]), "=r"(B[2]), "=r"(B[3]), "=r"(B[4]), "=r"(B[5]), "=r"(B[6]), "=r"(B[7]),
          "=r"(B[8])
        : "r"(x.l[1]), "r"(x.l[3]), "r"(x.l[5]), "r"(x.l[7]), "r"(y.l[0]));
    row_a(A, u.l, v.l[0]);
    row_b_nl(B, u.l, v.l[0]);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        if (i > 0) {
            row_b_z(A, B, L, x.l, y.l[i]);
            row_a(A, x.l, y.l[i]);
            row_b_nl(B, u.l, v.l[i]);
            row_a(A, u.l, v.l[i]);
        }
        uint32_t m = mont_m(A[0]);
        red_a(A, m);
        red_b(B, m);
        L = A[1];
        uint32_t nA[9], nB[9];
#pragma unroll
        for (int q = 0; q < 9; ++q) nA[q] = B[q];
#pragma unroll
        for (int q = 0; q < 7; ++q) nB[q] = A[q + 2];
        nB[7] = 0;
        nB[8] = 0;
#pragma unroll
        for (int q = 0; q < 9; ++q) { A[q] = nA[q]; B[q] = nB[q]; }
    }
    fe r;
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]), "=r"(r.l[6]),
          "=r"(r.l[7])
        : "r"(A[0]), "r"(A[1]), "r"(A[2]), "r"(A[3]), "r"(A[4]), "r"(A[5]), "r"(A[6]), "r"(A[7]),
          "r"(L), "r"(B[0]), "r"(B[1]), "r"(B[2]), "r"(B[3]), "r"(B[4]), "r"(B[5]), "r"(B[6]));
    return r;
}

// ---------------------------------------------------------------- fixed-multiplier product (folds)
//
// Every fold of one proof in one round multiplies by the SAME challenge r (Alg. 1
// line 5), so the product r * x can use a per-(proof, round) table instead of a CIOS product:
//   K_i = r * 2^(32 i + 64) mod p,  i = 0..7  (canonical, in shared memory, built once per CTA)
//   V   = sum_i x_i K_i   (x_i = 32-bit limbs of x; any x < 2^256)   ->  V < 8 * 2^32 * p < 2^289
//   two Montgomery word steps: (V + q p) / 2^64 == r x (mod p),  result < p (1 + 2^-29) < 2p.
// 64 + 18 limb products instead of 136 for mont_mul_lz (the rows need no reduction in between).

// 8 words of K_i from shared memory (broadcast).  The address carries a false data dependency on
// a word of the previous row (dep & zmask, zmask = 0 from a kernel parameter ptxas cannot see
// through), so the loads stay one row ahead instead of the whole 64-word table being hoisted into
// registers.
__device__ __forceinline__ void lds_k(uint32_t k[8], const fe *Ki, uint32_t dep, uint32_t zmask) {
    const uint32_t a = (uint32_t)__cvta_generic_to_shared(Ki) + (dep & zmask);
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%8];\n\t"
                 "ld.shared.v4.u32 {%4, %5, %6, %7}, [%8+16];"
                 : "=r"(k[0]), "=r"(k[1]), "=r"(k[2]), "=r"(k[3]), "=r"(k[4]), "=r"(k[5]), "=r"(k[6]), "=r"(k[7])
                 : "r"(a));
}

// carry-propagating add of a pending word at column 0 of A (A[q] at column q)
__device__ __forceinline__ void add_l(uint32_t A[9], uint32_t L) {
    asm("add.cc.u32  %0, %0, %9;\n\t"
        "addc.cc.u32 %1, %1, 0;\n\t"
        "addc.cc.u32 %2, %2, 0;\n\t"
        "addc.cc.u32 %3, %3, 0;\n\t"
        "addc.cc.u32 %4, %4, 0;\n\t"
        "addc.cc.u32 %5, %5, 0;\n\t"
        "addc.cc.u32 %6, %6, 0;\n\t"
        "addc.cc.u32 %7, %7, 0;\n\t"
        "addc.u32    %8, %8, 0;"
        : "+r"(A[0]), "+r"(A[1]), "+r"(A[2]), "+r"(A[3]), "+r"(A[4]), "+r"(A[5]), "+r"(A[6]), "+r"(A[7]),
          "+r"(A[8])
        : "r"(L));
}

__device__ __forceinline__ fe fixmul_lz(const fe &x, const fe *K, uint32_t zmask) {
    uint32_t A[9], B[9], k[8];
    lds_k(k, K, x.l[0], zmask);
    // row 0: A (columns 0..8) = K0_even * x0, B (columns 1..9) = K0_odd * x0
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(A[0]), "=r"(A[1]), "=r"(A[2]), "=r"(A[3]), "=r"(A[4]), "=r"(A[5]), "=r"(A[6]), "=r"(A[7]),
          "=r"(A[8])
        : "r"(k[0]), "r"(k[2]), "r"(k[4]), "r"(k[6]), "r"(x.l[0]));
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(B[0]), "=r"(B[1]), "=r"(B[2]), "=r"(B[3]), "=r"(B[4]), "=r"(B[5]), "=r"(B[6]), "=r"(B[7]),
          "=r"(B[8])
        : "r"(k[1]), "r"(k[3]), "r"(k[5]), "r"(k[7]), "r"(x.l[0]));
    // rows 1..7: every row lands on the same columns (K_i already carries the 2^(32 i) weight)
#pragma unroll
    for (int i = 1; i < 8; ++i) {
        lds_k(k, K + i, A[0], zmask);
        row_a(A, k, x.l[i]);
        row_b_nl(B, k, x.l[i]);
    }
    // two Montgomery word steps (divide by 2^64); same column bookkeeping as mont_mul_lz
    uint32_t L = 0;
#pragma unroll
    for (int s = 0; s < 2; ++s) {
        if (s > 0) add_l(A, L);
        const uint32_t m = mont_m(A[0]);
        red_a(A, m);
        red_b(B, m);
        L = A[1];
        uint32_t nA[9], nB[9];
#pragma unroll
        for (int q = 0; q < 9; ++q) nA[q] = B[q];
#pragma unroll
        for (int q = 0; q < 7; ++q) nB[q] = A[q + 2];
        nB[7] = 0;
        nB[8] = 0;
#pragma unroll
        for (int q = 0; q < 9; ++q) { A[q] = nA[q]; B[q] = nB[q]; }
    }
    fe r;   // A + L + (B << 32) < 2^255: A8, B7, B8 are zero
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]), "=r"(r.l[6]),
          "=r"(r.l[7])
        : "r"(A[0]), "r"(A[1]), "r"(A[2]), "r"(A[3]), "r"(A[4]), "r"(A[5]), "r"(A[6]), "r"(A[7]),
          "r"(L), "r"(B[0]), "r"(B[1]), "r"(B[2]), "r"(B[3]), "r"(B[4]), "r"(B[5]), "r"(B[6]));
    return r;
}

// (x*y + u*v) * R^{-1} mod p, canonical; x, y, u, v canonical (result of the lazy form < 3p)
__device__ __forceinline__ fe mont_mul2(const fe &x, const fe &y, const fe &u, const fe &v) {
    return fe_reduce_once(fe_reduce_once(mont_mul2_lz(x, y, u, v)));
}

// ---------------------------------------------------------------- lazy ("< 2p") arithmetic
// Hot-loop values are kept in [0, 2p) instead of [0, p); every bound below uses 4p < 2^256.

// 2p (LE 32-bit limbs)
#define BZK_2P0 0xe0000002u
#define BZK_2P1 0x87c3eb27u
#define BZK_2P2 0xf372e122u
#define BZK_2P3 0x5067d090u
#define BZK_2P4 0x0302b0bau
#define BZK_2P5 0x70a08b6du
#define BZK_2P6 0xc2634053u
#define BZK_2P7 0x60c89ce5u

// b + 2p - a  (a, b < 2p -> result in (0, 4p)); branch-free
__device__ __forceinline__ fe lz_sub(const fe &b, const fe &a) {
    fe t, r;
    asm("sub.cc.u32  %0, %8,  %16;\n\t"
        "subc.cc.u32 %1, %9,  %17;\n\t"
        "subc.cc.u32 %2, %10, %18;\n\t"
        "subc.cc.u32 %3, %11, %19;\n\t"
        "subc.cc.u32 %4, %12, %20;\n\t"
        "subc.cc.u32 %5, %13, %21;\n\t"
        "subc.cc.u32 %6, %14, %22;\n\t"
        "subc.u32    %7, %15, %23;"
        : "=r"(t.l[0]), "=r"(t.l[1]), "=r"(t.l[2]), "=r"(t.l[3]), "=r"(t.l[4]), "=r"(t.l[5]), "=r"(t.l[6]),
          "=r"(t.l[7])
        : "n"(BZK_2P0), "n"(BZK_2P1), "n"(BZK_2P2), "n"(BZK_2P3), "n"(BZK_2P4), "n"(BZK_2P5), "n"(BZK_2P6),
          "n"(BZK_2P7), "r"(a.l[0]), "r"(a.l[1]), "r"(a.l[2]), "r"(a.l[3]), "r"(a.l[4]), "r"(a.l[5]), "r"(a.l[6]),
          "r"(a.l[7]));
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]), "=r"(r.l[6]),
          "=r"(r.l[7])
        : "r"(t.l[0]), "r"(t.l[1]), "r"(t.l[2]), "r"(t.l[3]), "r"(t.l[4]), "r"(t.l[5]), "r"(t.l[6]), "r"(t.l[7]),
          "r"(b.l[0]), "r"(b.l[1]), "r"(b.l[2]), "r"(b.l[3]), "r"(b.l[4]), "r"(b.l[5]), "r"(b.l[6]), "r"(b.l[7]));
    return r;
}

// x < 4p  ->  x mod 2p-range: subtract 2p when x >= 2p (result < 2p)
__device__ __forceinline__ fe lz_red(const fe &x) {
    fe s;
    uint32_t borrow;
    asm("sub.cc.u32  %0, %9,  %17;\n\t"
        "subc.cc.u32 %1, %10, %18;\n\t"
        "subc.cc.u32 %2, %11, %19;\n\t"
        "subc.cc.u32 %3, %12, %20;\n\t"
        "subc.cc.u32 %4, %13, %21;\n\t"
        "subc.cc.u32 %5, %14, %22;\n\t"
        "subc.cc.u32 %6, %15, %23;\n\t"
        "subc.cc.u32 %7, %16, %24;\n\t"
        "subc.u32    %8, 0, 0;"
        : "=r"(s.l[0]), "=r"(s.l[1]), "=r"(s.l[2]), "=r"(s.l[3]), "=r"(s.l[4]), "=r"(s.l[5]),
          "=r"(s.l[6]), "=r"(s.l[7]), "=r"(borrow)
        : "r"(x.l[0]), "r"(x.l[1]), "r"(x.l[2]), "r"(x.l[3]), "r"(x.l[4]), "r"(x.l[5]), "r"(x.l[6]),
          "r"(x.l[7]), "n"(BZK_2P0), "n"(BZK_2P1), "n"(BZK_2P2), "n"(BZK_2P3), "n"(BZK_2P4), "n"(BZK_2P5),
          "n"(BZK_2P6), "n"(BZK_2P7));
    fe r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.l[i] = borrow ? x.l[i] : s.l[i];
    return r;
}

// plain 256-bit add (caller guarantees no overflow, e.g. a < 2p, b < 2p)
__device__ __forceinline__ fe lz_add(const fe &a, const fe &b) {
    fe s;
    asm("add.cc.u32  %0, %8,  %16;\n\t"
        "addc.cc.u32 %1, %9,  %17;\n\t"
        "addc.cc.u32 %2, %10, %18;\n\t"
        "addc.cc.u32 %3, %11, %19;\n\t"
        "addc.cc.u32 %4, %12, %20;\n\t"
        "addc.cc.u32 %5, %13, %21;\n\t"
        "addc.cc.u32 %6, %14, %22;\n\t"
        "addc.u32    %7, %15, %23;"
        : "=r"(s.l[0]), "=r"(s.l[1]), "=r"(s.l[2]), "=r"(s.l[3]), "=r"(s.l[4]), "=r"(s.l[5]),
          "=r"(s.l[6]), "=r"(s.l[7])
        : "r"(a.l[0]), "r"(a.l[1]), "r"(a.l[2]), "r"(a.l[3]), "r"(a.l[4]), "r"(a.l[5]), "r"(a.l[6]),
          "r"(a.l[7]), "r"(b.l[0]), "r"(b.l[1]), "r"(b.l[2]), "r"(b.l[3]), "r"(b.l[4]), "r"(b.l[5]),
          "r"(b.l[6]), "r"(b.l[7]));
    return s;
}

// 288-bit accumulator for sums of lazy products (each < 3p): 8 limbs + a carry word
struct acc9 { fe lo; uint32_t hi; };
__device__ __forceinline__ acc9 acc9_zero() { acc9 a; a.lo = fe_zero(); a.hi = 0; return a; }
__device__ __forceinline__ void acc9_add(acc9 &a, const fe &x) {
    asm("add.cc.u32  %0, %0, %9;\n\t"
        "addc.cc.u32 %1, %1, %10;\n\t"
        "addc.cc.u32 %2, %2, %11;\n\t"
        "addc.cc.u32 %3, %3, %12;\n\t"
        "addc.cc.u32 %4, %4, %13;\n\t"
        "addc.cc.u32 %5, %5, %14;\n\t"
        "addc.cc.u32 %6, %6, %15;\n\t"
        "addc.cc.u32 %7, %7, %16;\n\t"
        "addc.u32    %8, %8, 0;"
        : "+r"(a.lo.l[0]), "+r"(a.lo.l[1]), "+r"(a.lo.l[2]), "+r"(a.lo.l[3]), "+r"(a.lo.l[4]), "+r"(a.lo.l[5]),
          "+r"(a.lo.l[6]), "+r"(a.lo.l[7]), "+r"(a.hi)
        : "r"(x.l[0]), "r"(x.l[1]), "r"(x.l[2]), "r"(x.l[3]), "r"(x.l[4]), "r"(x.l[5]), "r"(x.l[6]), "r"(x.l[7]));
}

// ---------------------------------------------------------------- unreduced product sums
//
// A round sum  S = sum_j x_j y_j  needs only ONE Montgomery reduction per thread, after the loop:
// the 512-bit products are added into a 544-bit accumulator (17 words; room for 2^32 products of
// values < 4p) and acc17_to_fe returns S * R^{-1} mod p -- the same value (and scale) as summing
// mont_mul(x_j, y_j).  64 limb products per product instead of 100 (mont_mul2) or 136 (mont_mul).
struct acc17 { uint32_t w[17]; };
__device__ __forceinline__ acc17 acc17_zero() {
    acc17 a;
#pragma unroll
    for (int i = 0; i < 17; ++i) a.w[i] = 0;
    return a;
}

// acc += x * y   (x * y < 2^512).  Row-scanned product on the parity-aligned A/B chains of
// mont_mul_lz without the reduction rows: after row i the lowest relative column (A0) is final
// and is emitted to out[i]; the shift re-pairs the chains exactly as in mont_mul_lz.
__device__ __forceinline__ void mul_acc(acc17 &acc, const fe &x, const fe &y) {
    uint32_t A[9], B[9], L, out[8];
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(A[0]), "=r"(A[1]), "=r"(A[2]), "=r"(A[3]), "=r"(A[4]), "=r"(A[5]), "=r"(A[6]), "=r"(A[7]),
          "=r"(A[8])
        : "r"(x.l[0]), "r"(x.l[2]), "r"(x.l[4]), "r"(x.l[6]), "r"(y.l[0]));
    asm("mul.lo.u32 %0, %9,  %13;\n\t"
        "mul.hi.u32 %1, %9,  %13;\n\t"
        "mul.lo.u32 %2, %10, %13;\n\t"
        "mul.hi.u32 %3, %10, %13;\n\t"
        "mul.lo.u32 %4, %11, %13;\n\t"
        "mul.hi.u32 %5, %11, %13;\n\t"
        "mul.lo.u32 %6, %12, %13;\n\t"
        "mul.hi.u32 %7, %12, %13;\n\t"
        "mov.u32    %8, 0;"
        : "=r"(B[0]), "=r"(B[1]), "=r"(B[2]), "=r"(B[3]), "=r"(B[4]), "=r"(B[5]), "=r"(B[6]), "=r"(B[7]),
          "=r"(B[8])
        : "r"(x.l[1]), "r"(x.l[3]), "r"(x.l[5]), "r"(x.l[7]), "r"(y.l[0]));
#pragma unroll
    for (int i = 1; i < 8; ++i) {
        out[i - 1] = A[0];
        L = A[1];
        uint32_t nA[9], nB[9];
#pragma unroll
        for (int q = 0; q < 9; ++q) nA[q] = B[q];
#pragma unroll
        for (int q = 0; q < 7; ++q) nB[q] = A[q + 2];
        nB[7] = 0;
        nB[8] = 0;
#pragma unroll
        for (int q = 0; q < 9; ++q) { A[q] = nA[q]; B[q] = nB[q]; }
        row_b_z(A, B, L, x.l, y.l[i]);
        row_a(A, x.l, y.l[i]);
    }
    out[7] = A[0];
    // acc[0..7] += out, acc[8..15] += A[1..8], carry -> acc[16]; then acc[8..16] += B[0..8]
    asm("add.cc.u32  %0,  %0,  %17;\n\t"
        "addc.cc.u32 %1,  %1,  %18;\n\t"
        "addc.cc.u32 %2,  %2,  %19;\n\t"
        "addc.cc.u32 %3,  %3,  %20;\n\t"
        "addc.cc.u32 %4,  %4,  %21;\n\t"
        "addc.cc.u32 %5,  %5,  %22;\n\t"
        "addc.cc.u32 %6,  %6,  %23;\n\t"
        "addc.cc.u32 %7,  %7,  %24;\n\t"
        "addc.cc.u32 %8,  %8,  %25;\n\t"
        "addc.cc.u32 %9,  %9,  %26;\n\t"
        "addc.cc.u32 %10, %10, %27;\n\t"
        "addc.cc.u32 %11, %11, %28;\n\t"
        "addc.cc.u32 %12, %12, %29;\n\t"
        "addc.cc.u32 %13, %13, %30;\n\t"
        "addc.cc.u32 %14, %14, %31;\n\t"
        "addc.cc.u32 %15, %15, %32;\n\t"
        "addc.u32    %16, %16, 0;"
        : "+r"(acc.w[0]), "+r"(acc.w[1]), "+r"(acc.w[2]), "+r"(acc.w[3]), "+r"(acc.w[4]), "+r"(acc.w[5]),
          "+r"(acc.w[6]), "+r"(acc.w[7]), "+r"(acc.w[8]), "+r"(acc.w[9]), "+r"(acc.w[10]), "+r"(acc.w[11]),
          "+r"(acc.w[12]), "+r"(acc.w[13]), "+r"(acc.w[14]), "+r"(acc.w[15]), "+r"(acc.w[16])
        : "r"(out[0]), "r"(out[1]), "r"(out[2]), "r"(out[3]), "r"(out[4]), "r"(out[5]), "r"(out[6]), "r"(out[7]),
          "r"(A[1]), "r"(A[2]), "r"(A[3]), "r"(A[4]), "r"(A[5]), "r"(A[6]), "r"(A[7]), "r"(A[8]));
    asm("add.cc.u32  %0, %0, %9;\n\t"
        "addc.cc.u32 %1, %1, %10;\n\t"
        "addc.cc.u32 %2, %2, %11;\n\t"
        "addc.cc.u32 %3, %3, %12;\n\t"
        "addc.cc.u32 %4, %4, %13;\n\t"
        "addc.cc.u32 %5, %5, %14;\n\t"
        "addc.cc.u32 %6, %6, %15;\n\t"
        "addc.cc.u32 %7, %7, %16;\n\t"
        "addc.u32    %8, %8, %17;"
        : "+r"(acc.w[8]), "+r"(acc.w[9]), "+r"(acc.w[10]), "+r"(acc.w[11]), "+r"(acc.w[12]), "+r"(acc.w[13]),
          "+r"(acc.w[14]), "+r"(acc.w[15]), "+r"(acc.w[16])
        : "r"(B[0]), "r"(B[1]), "r"(B[2]), "r"(B[3]), "r"(B[4]), "r"(B[5]), "r"(B[6]), "r"(B[7]), "r"(B[8]));
}

__device__ __forceinline__ fe fe_const(int which) {
    fe r;
    switch (which) {
        case 1: {  // R mod p
            const uint32_t v[8] = {0x4ffffffbu, 0xac96341cu, 0x9f60cd29u, 0x36fc7695u,
                                   0x7879462eu, 0x666ea36fu, 0x9a07df2fu, 0x0e0a77c1u};
            _Pragma("unroll") for (int i = 0; i < 8; ++i) r.l[i] = v[i];
            break;
        }
        case 2: {  // R^2 mod p
            const uint32_t v[8] = {0xae216da7u, 0x1bb8e645u, 0xe35c59e3u, 0x53fe3ab1u,
                                   0x53bb8085u, 0x8c49833du, 0x7f4e44a5u, 0x0216d0b1u};
            _Pragma("unroll") for (int i = 0; i < 8; ++i) r.l[i] = v[i];
            break;
        }
        case 3: {  // R^3 mod p
            const uint32_t v[8] = {0xb4bf0040u, 0x5e94d8e1u, 0x1cfbb6b8u, 0x2a489cbeu,
                                   0xa19fcfedu, 0x893cc664u, 0x7fcc657cu, 0x0cf8594bu};
            _Pragma("unroll") for (int i = 0; i < 8; ++i) r.l[i] = v[i];
            break;
        }
        default: r = fe_zero(); r.l[0] = 1; break;
    }
    return r;
}

// x^e for small fixed powers of R: R^d mod p = mont_mul chain of R^2 and R^3 (computed once per use)
//   R^4 = mont_mul(R^3, R^2);  R^5 = mont_mul(R^4, R^2)  (mont_mul(R^a, R^b) = R^{a+b-1})
__device__ __forceinline__ fe fe_R_pow(int d) {
    if (d <= 1) return fe_const(1);
    if (d == 2) return fe_const(2);
    if (d == 3) return fe_const(3);
    fe r = fe_const(3);
    for (int e = 3; e < d; ++e) r = mont_mul(r, fe_const(2));
    return r;
}

// canonicalise an arbitrary 256-bit value (< 2^256 < 6p): subtract p up to 5 times
__device__ __forceinline__ fe fe_reduce_256(const fe &a) {
    fe r = a;
#pragma unroll 1
    for (int it = 0; it < 6; ++it) {
        fe s;
        uint32_t borrow = sub_p(s, r);
        if (borrow) break;
        r = s;
    }
    return r;
}

__device__ __forceinline__ bool fe_is_canon(const fe &a) {
    fe s;
    return sub_p(s, a) != 0;
}

// ---------------------------------------------------------------- memory helpers

// 32-byte element load/store as two 128-bit accesses (coalesced across a warp)
__device__ __forceinline__ fe ld_fe(const fe *p) {
    const uint4 *q = reinterpret_cast<const uint4 *>(p);
    uint4 x = __ldg(q), y = __ldg(q + 1);
    fe r;
    r.l[0] = x.x; r.l[1] = x.y; r.l[2] = x.z; r.l[3] = x.w;
    r.l[4] = y.x; r.l[5] = y.y; r.l[6] = y.z; r.l[7] = y.w;
    return r;
}

// 256-bit global accesses (sm_100: LDG/STG.E.ENL2.256): one instruction per element, and every
// store writes whole 32-byte sectors (with two 128-bit stores per element the fused rounds read
// ~60 % of their written bytes back from DRAM: partial-sector write fills, ncu r01g)
#define BZK_LD8(MOD, r, ptr)                                                                      \
    asm("ld.global" MOD ".v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"                          \
        : "=r"((r).l[0]), "=r"((r).l[1]), "=r"((r).l[2]), "=r"((r).l[3]), "=r"((r).l[4]), "=r"((r).l[5]), \
          "=r"((r).l[6]), "=r"((r).l[7])                                                            \
        : "l"(ptr))

// streaming load for data read exactly once (evict-first)
__device__ __forceinline__ fe ld_fe_stream(const fe *p) {
    fe r;
    BZK_LD8(".cs", r, p);
    return r;
}

// L2-coherent load (data written by other CTAs of the same launch)
__device__ __forceinline__ fe ld_fe_cg(const fe *p) {
    const uint4 *q = reinterpret_cast<const uint4 *>(p);
    uint4 x = __ldcg(q), y = __ldcg(q + 1);
    fe r;
    r.l[0] = x.x; r.l[1] = x.y; r.l[2] = x.z; r.l[3] = x.w;
    r.l[4] = y.x; r.l[5] = y.y; r.l[6] = y.z; r.l[7] = y.w;
    return r;
}

__device__ __forceinline__ void st_fe(fe *p, const fe &v) {
    asm volatile("st.global.v8.u32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(p), "r"(v.l[0]), "r"(v.l[1]),
                 "r"(v.l[2]), "r"(v.l[3]), "r"(v.l[4]), "r"(v.l[5]), "r"(v.l[6]), "r"(v.l[7])
                 : "memory");
}

__device__ __forceinline__ void st_fe_cg(fe *p, const fe &v) {
    uint4 *q = reinterpret_cast<uint4 *>(p);
    __stcg(q, make_uint4(v.l[0], v.l[1], v.l[2], v.l[3]));
    __stcg(q + 1, make_uint4(v.l[4], v.l[5], v.l[6], v.l[7]));
}

__device__ __forceinline__ fe shfl_down_fe(const fe &v, int delta) {
    fe r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.l[i] = __shfl_down_sync(0xffffffffu, v.l[i], delta);
    return r;
}

}  // namespace bzk
