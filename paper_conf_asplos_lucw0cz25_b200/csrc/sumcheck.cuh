// sumcheck.cuh -- the batched sum-check round kernels.
//
// One proof = d multilinear tables of 2^k BN254-Fr elements, layout [B][d][2^k] x 32 B.
// Per round i (h = 2^{k-i} pairs), following PAPER.md:111 (Alg. 1) generalised to a product of
// d multilinears with Fiat-Shamir challenges (north_star; readings R3-R8 in DESIGN.md):
//     g_i(t) = sum_{j<h} prod_m (a_mj + t (b_mj - a_mj)),  t = 0..d
//     (a, b) = (T[2j], T[2j+1]) for LSB order, (T[j], T[j+h]) for MSB order (Alg. 1)
//     r_i    = SHA-256 transcript -> F_p
//     T'[j]  = a + r_i (b - a)
//
// Kernels (B200 re-design of the paper's "one kernel per round"):
//   k_round<D,ORDER,FIRST>  rounds with h > tail threshold, all proofs of a wave in lockstep.
//       FIRST : round 1, evaluation only (reads the input once), every point t = 0..d.
//       !FIRST: fused fold(r_{i-1}) + eval(i): a thread reads 4 entries per table, writes the 2
//               folded ones to the other ping-pong buffer (Fig. 5) and evaluates round i
//               on them in registers (the sums reuse the update's loads).  g_i(1) is not
//               summed: it is derived exactly as claim_i - g_i(0), claim_i = g_{i-1}(r_{i-1}).
//       The last product of every summed point goes unreduced into a 544-bit per-thread
//       accumulator (mul_acc) and is reduced once after the loop.  Partial sums: per thread -> warp shuffle -> shared memory ->
//       per-CTA partial in global -> last-CTA ticket; the last CTA of each proof reduces the
//       partials, hashes the transcript and publishes r_i (single pass, no extra launch; the
//       paper's reduction made repeated global passes).
//   k_tail<D,ORDER>  one CTA per proof finishes the remaining rounds (h <= tail threshold) in
//       shared memory, including the final fold that yields final_m = f_m(rho).
#pragma once
#include <cooperative_groups.h>
#include <cuda.h>
#include <stdint.h>
#include "field.cuh"

#ifndef BZK_RT
#define BZK_RT 256        // threads per CTA of k_round
#endif
#ifndef BZK_ROUND_OCC
#define BZK_ROUND_OCC 2   // resident CTAs per SM requested for k_round (d <= 2)
#endif
#include "sha256.cuh"

// BZK_CHECK builds (scripts/gpu_r02chk.sh; compute-sanitizer is closed on the GPU pool): device-side
// asserts on the hot path's indices -- pair index within the round, partial slot within the proof's
// CTAs, shared-memory tiles and slots within the launch's dynamic shared memory.  A failed check traps
// (the call returns BZK_ECUDA).  Compiled out otherwise.
#ifdef BZK_CHECK
#define BZK_ASSERT(...) do { if (!(__VA_ARGS__)) __trap(); } while (0)
#else
#define BZK_ASSERT(...) do { } while (0)
#endif

namespace bzk {

struct ProofState {
    uint32_t st[8];   // transcript state_i
    fe rmont;         // r_i * R mod p (Montgomery) for the next fold
    fe claim;         // claim_{i+1} = g_i(r_i) (standard form)
};

// Device constants (filled once per context by k_init_consts):
//   [0..4]        l * R mod p, l = 0..4          (Montgomery form of the node l)
//   [5 + 5D + j]  w_{D,j}^{-1} * R mod p, w_{D,j} = prod_{l != j, 0<=l<=D} (j - l)   (Lagrange)
//   [30 + i]      2^(32 i + 64) mod p, i = 0..7   (fixed-multiplier fold table: K_i = r * this)
constexpr int kConstLR = 0;
constexpr int kConstInvW = 5;
constexpr int kConstPow2 = 30;
constexpr int kNumConsts = 5 + 5 * 5 + 8;

struct RoundParams {
    const fe *src;        // FIRST: [Bw][D][2h]; else [Bw][D][4h]
    fe *dst;              // !FIRST: [Bw][D][2h]
    uint32_t log_h;       // h = 2^log_h pairs per proof this round
    uint32_t round;       // i, 1-based
    uint32_t k, order;
    uint32_t ctas;        // CTAs per proof
    fe *partials;         // [Bw][ctas][D+1]
    uint32_t *tickets;    // [Bw]
    ProofState *ps;       // [Bw]
    fe *round_evals;      // [Bw][k][D+1]
    fe *challenges;       // [Bw][k]
    fe *claims;           // [Bw] (may be null)
    const fe *consts;     // kNumConsts
    uint32_t given;       // 1: challenges are inputs (BZK_F_GIVEN_CHALLENGES), no transcript
    uint32_t cluster;     // thread-block cluster size along x (1 = none); divides ctas
    uint32_t zero;        // always 0 (opaque to the compiler: orders the fold-table loads, fixmul_lz)
    uint32_t tma;         // 1: operands staged into shared memory by TMA (k_round<..., TMA = true>)
};

// ---------------------------------------------------------------- reductions

template <int V>
__device__ __forceinline__ void warp_reduce(fe (&acc)[V]) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = fe_add(acc[v], shfl_down_fe(acc[v], off));
}

// Block-wide sum of V field elements; result valid in thread 0. smem: [32][V] fe.
template <int V>
__device__ __forceinline__ void block_reduce(fe (&acc)[V], fe *smem) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = (blockDim.x + 31) >> 5;
    warp_reduce<V>(acc);
    if (lane == 0)
#pragma unroll
        for (int v = 0; v < V; ++v) smem[warp * V + v] = acc[v];
    __syncthreads();
    if (warp == 0) {
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = lane < nwarps ? smem[lane * V + v] : fe_zero();
        warp_reduce<V>(acc);
    }
    __syncthreads();
}

// ---------------------------------------------------------------- per-pair math

// Summed evaluation points of the global round kernels (the "infinity" point is the leading
// coefficient of g_i, i.e. the sum of prod_m delta_m -- it replaces t = d and needs no additions):
//   FIRST  (round 1)        : t = 0, 1, ..., d-1, inf          (d = 1: t = 0, 1)
//   DERIVE (fused rounds)   : t = 0, 2, ..., d-1, inf          (d = 1: t = 0); g(1) = claim - g(0)
// finalize_round() rebuilds g(d) = sum_{j<d} (-1)^{d-1-j} C(d,j) g(j) + d! * c_inf.
template <int D, bool DERIVE> struct Pts { static constexpr int NV = DERIVE ? D : D + 1; };

template <int D, bool DERIVE>
__device__ __forceinline__ constexpr int point_t(int idx) {   // -1 = infinity
    if (D == 1) return idx;
    if (idx == Pts<D, DERIVE>::NV - 1) return -1;
    return DERIVE ? (idx == 0 ? 0 : idx + 1) : idx;
}

// d = 1: g(t) is a sum of table values only (no products), so a pair's points t = 0 (a) and, in
// round 1, t = 1 (b) are summed straight into 288-bit accumulators; the fused rounds derive g(1).
// Two pairs are added together first (lazy values < 2p each).
template <int D, bool DERIVE>
__device__ __forceinline__ void eval_two(const fe (&a)[D], const fe (&s)[D], const fe (&a2)[D], const fe (&s2)[D],
                                         acc9 (&acc)[Pts<D, DERIVE>::NV]) {
    static_assert(D == 1, "d >= 2 sums go through eval_one / mul_acc");
    acc9_add(acc[0], lz_add(a[0], a2[0]));
    if (!DERIVE) acc9_add(acc[1], lz_add(s[0], s2[0]));   // round 1: s = b
}

// 288-bit accumulator -> canonical field element: hi * 2^256 + lo = hi * (R mod p) + lo (mod p)
__device__ __forceinline__ fe acc9_to_fe(const acc9 &a) {
    fe h = fe_zero();
    h.l[0] = a.hi;
    return fe_add(fe_reduce_256(a.lo), mont_mul(h, fe_const(2)));   // hi * R^2 * R^-1 = hi * R
}

// 544-bit accumulator -> S * 2^-288 mod p, canonical: NINE Montgomery word steps, so the quotient
// W = (S + q p) / 2^288 < 2^256 + p needs one conditional subtraction and no extra product (the
// 8-step form below leaves a 2^256 "hi" part that costs a full Montgomery product).  Callers fold
// the extra 2^-32 into a constant (k_multi: weights w 2^288 mod p).
__device__ __forceinline__ fe acc17_to_fe_288(const acc17 &a) {
    const uint32_t P[8] = {BZK_P0, BZK_P1, BZK_P2, BZK_P3, BZK_P4, BZK_P5, BZK_P6, BZK_P7};
    uint32_t t[18];
#pragma unroll
    for (int i = 0; i < 17; ++i) t[i] = a.w[i];
    t[17] = 0;
#pragma unroll
    for (int i = 0; i < 9; ++i) {
        const uint32_t m = t[i] * BZK_NP0;
        uint64_t c = 0;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint64_t x = (uint64_t)m * P[j] + t[i + j] + c;
            t[i + j] = (uint32_t)x;
            c = x >> 32;
        }
#pragma unroll
        for (int j = i + 8; j < 18; ++j) {
            const uint64_t x = (uint64_t)t[j] + c;
            t[j] = (uint32_t)x;
            c = x >> 32;
        }
    }
    fe w;
#pragma unroll
    for (int i = 0; i < 8; ++i) w.l[i] = t[9 + i];
    if (t[17]) {   // W >= 2^256: W - p < 2^256 (W < 2^256 + p); the borrow out of the top word cancels t[17]
        fe r;
        sub_p(r, w);
        w = r;
    }
    return fe_reduce_256(w);
}

// 544-bit accumulator -> S * R^{-1} mod p, canonical (once per thread after the loop; plain code)
__device__ __forceinline__ fe acc17_to_fe(const acc17 &a) {
    const uint32_t P[8] = {BZK_P0, BZK_P1, BZK_P2, BZK_P3, BZK_P4, BZK_P5, BZK_P6, BZK_P7};
    uint32_t t[18];
#pragma unroll
    for (int i = 0; i < 17; ++i) t[i] = a.w[i];
    t[17] = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {   // Montgomery REDC: t += m p 2^(32 i) clears word i
        const uint32_t m = t[i] * BZK_NP0;
        uint64_t c = 0;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint64_t x = (uint64_t)m * P[j] + t[i + j] + c;
            t[i + j] = (uint32_t)x;
            c = x >> 32;
        }
#pragma unroll
        for (int j = i + 8; j < 18; ++j) {
            const uint64_t x = (uint64_t)t[j] + c;
            t[j] = (uint32_t)x;
            c = x >> 32;
        }
    }
    // W = t[8..17] = (S + q p) / R < 2^288 + p:  W = lo + hi 2^256,  hi 2^256 = mont_mul(hi, R^2)
    fe lo, hi = fe_zero();
#pragma unroll
    for (int i = 0; i < 8; ++i) lo.l[i] = t[8 + i];
    hi.l[0] = t[16];
    hi.l[1] = t[17];
    return fe_add(fe_reduce_256(lo), mont_mul(hi, fe_const(2)));
}

// d >= 2: the last product of every summed point goes into a 544-bit accumulator (mul_acc) and is
// reduced once per thread (d = 1 has no products: its sums go through eval_two's 288-bit adds).

// one pair at the summed points (same point sets and lazy bounds as eval_two)
template <int D, bool DERIVE>
__device__ __forceinline__ void eval_one(const fe (&a)[D], const fe (&s)[D], acc17 (&acc)[Pts<D, DERIVE>::NV]) {
    constexpr int NV = Pts<D, DERIVE>::NV;
    fe v[D], dl[D];
#pragma unroll
    for (int idx = 0; idx < NV; ++idx) {
        const int t = point_t<D, DERIVE>(idx);
        if ((t < 0 || t == 2) && !DERIVE) {   // round 1: delta = b - a on demand
#pragma unroll
            for (int m = 0; m < D; ++m) {
                dl[m] = lz_sub(s[m], a[m]);
                if (!(D == 2 && m == 0)) dl[m] = lz_red(dl[m]);
            }
        }
        const fe *x;
        if (t == 0) x = a;
        else if (t == 1) x = s;                                    // FIRST only: s = b
        else if (t < 0) x = DERIVE ? s : dl;
        else {
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const fe &d1 = DERIVE ? s[m] : dl[m];
                if (t == 2) {
                    v[m] = lz_red(lz_add(DERIVE ? a[m] : s[m], d1));
                    if (DERIVE) v[m] = lz_red(lz_add(v[m], d1));
                } else {
                    v[m] = lz_red(lz_add(v[m], d1));
                }
            }
            x = v;
        }
        fe p = x[0];
#pragma unroll
        for (int m = 1; m < D - 1; ++m) p = mont_mul_lz(p, x[m]);
        mul_acc(acc[idx], p, x[D - 1]);
    }
}

// single pair, every point t = 0..D (used by the on-chip tail)
template <int D>
__device__ __forceinline__ void eval_pair(const fe (&a)[D], const fe (&b)[D], fe (&acc)[D + 1]) {
    fe v[D], delta[D];
#pragma unroll
    for (int m = 0; m < D; ++m) { v[m] = a[m]; delta[m] = fe_sub(b[m], a[m]); }
#pragma unroll
    for (int t = 0; t <= D; ++t) {
        if (t == 1) {
#pragma unroll
            for (int m = 0; m < D; ++m) v[m] = b[m];
        } else if (t > 1) {
#pragma unroll
            for (int m = 0; m < D; ++m) v[m] = fe_add(v[m], delta[m]);
        }
        fe prod = v[0];
#pragma unroll
        for (int m = 1; m < D; ++m) prod = mont_mul(prod, v[m]);
        acc[t] = fe_add(acc[t], prod);
    }
}

__device__ __forceinline__ fe fold1(const fe &a, const fe &b, const fe &rmont) {
    return fe_add(a, mont_mul(rmont, fe_sub(b, a)));
}

// lazy fold for the hot loop: a, b < 2p -> a + r (b - a) (mod p), result < 2p, through the
// fixed-multiplier table K of r (field.cuh fixmul_lz; K in shared memory)
__device__ __forceinline__ fe fold_fx(const fe &a, const fe &b, const fe *K, uint32_t zmask) {
    return lz_red(lz_add(a, fixmul_lz(lz_sub(b, a), K, zmask)));
}

// fused-round folds use the per-(proof, round) table K_i = r 2^(32i+64) (fixmul_lz)
#define BZK_FOLD(a, b) fold_fx(a, b, sK, zmask)

// ---------------------------------------------------------------- per-round finalisation

// x * c for a small non-negative integer c (finalisation only)
__device__ __forceinline__ fe fe_mul_small(const fe &x, int c) {
    fe r = fe_zero(), y = x;
    for (; c; c >>= 1) {
        if (c & 1) r = fe_add(r, y);
        y = fe_add(y, y);
    }
    return r;
}

// g(D) from g(0..D-1) and the leading coefficient c_inf:  sum_j (-1)^{D-1-j} C(D,j) g(j) + D! c_inf
template <int D>
__device__ __forceinline__ fe extrapolate_top(const fe (&g)[D + 1], const fe &cinf) {
    int binom = 1, fact = 1;
    fe pos = fe_zero(), neg = fe_zero();
    for (int j = 0; j < D; ++j) {
        const fe term = fe_mul_small(g[j], binom);
        if (((D - 1 - j) & 1) == 0) pos = fe_add(pos, term); else neg = fe_add(neg, term);
        binom = binom * (D - j) / (j + 1);
    }
    for (int j = 2; j <= D; ++j) fact *= j;
    return fe_add(fe_sub(pos, neg), fe_mul_small(cinf, fact));
}

// Fix the R^{-(D-1)} scale of the round sums, rebuild g(0..D), absorb g into the transcript,
// derive r_i, write the round's outputs and the next claim.  ONE thread per proof.
//   MODE 0: S holds g(0..D) directly, already in standard form (on-chip tail: its tables 1..D-1 are
//           held in Montgomery form, so the products carry no R^{-(D-1)})
//   MODE 1: S holds the FIRST point set, MODE 2 the DERIVE point set (see Pts / point_t)
// The next claim g_i(r_i) (global rounds) is NOT computed here: the caller's warp does the Lagrange
// sum with one lane per node (lagrange_warp), from g_out and the returned r R.
template <int D, int MODE>
__device__ __forceinline__ void finalize_round(fe (&S)[MODE == 2 ? D : D + 1], uint32_t round, ProofState &ps,
                                               fe *round_evals, fe *challenges, fe *claims, fe *rmont_out,
                                               fe *g_out, bool given) {
    constexpr int NS = MODE == 2 ? D : D + 1;
    fe g[D + 1];
    fe fixd[NS];
    if (MODE == 0) {
#pragma unroll
        for (int i = 0; i < NS; ++i) fixd[i] = S[i];
    } else {
        const fe RD = fe_R_pow(D);
#pragma unroll
        for (int i = 0; i < NS; ++i) fixd[i] = mont_mul_serial(S[i], RD);
    }
    if (MODE == 0) {
#pragma unroll
        for (int t = 0; t <= D; ++t) g[t] = fixd[t];
    } else {
        constexpr bool DERIVE = MODE == 2;
#pragma unroll
        for (int idx = 0; idx < NS; ++idx) {
            const int t = point_t<D, DERIVE>(idx);
            if (t >= 0) g[t] = fixd[idx];
        }
        if (DERIVE) g[1] = fe_sub(ps.claim, g[0]);
        if (D >= 2) g[D] = extrapolate_top<D>(g, fixd[NS - 1]);
    }
    fe r;
    if (given) {
        // paper-literal mode (Alg. 1: r_1..r_n are inputs): the challenge is read, not hashed
        r = ld_fe(&challenges[round - 1]);
    } else {
        uint32_t st[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) st[i] = ps.st[i];
        r = transcript_round_t<D>(st, g);
#pragma unroll
        for (int i = 0; i < 8; ++i) ps.st[i] = st[i];
        st_fe(&challenges[round - 1], r);
    }
#pragma unroll
    for (int t = 0; t <= D; ++t) st_fe(&round_evals[(size_t)(round - 1) * (D + 1) + t], g[t]);
    if (round == 1 && claims) st_fe(claims, fe_add(g[0], g[1]));
    fe rm = mont_mul_serial(r, fe_const(2));
    ps.rmont = rm;
    if (rmont_out) *rmont_out = rm;
    if (g_out)
#pragma unroll
        for (int t = 0; t <= D; ++t) g_out[t] = g[t];
}

// next claim g_i(r_i) = sum_j g_j / w_j * prod_{l != j} (r - l)  (Lagrange on the nodes 0..D): lane j
// of the calling warp computes term j (D + 1 serial products instead of (D + 1)^2), then a shuffle sum.
// Every lane of the warp calls it; g and rm in shared memory (written by lane 0 before a __syncwarp).
template <int D>
__device__ __forceinline__ fe lagrange_warp(const fe *g, const fe &rm, const fe *consts) {
    const int lane = threadIdx.x & 31;
    fe term = fe_zero();
    if (lane <= D) {
        term = mont_mul_serial(g[lane], consts[kConstInvW + 5 * D + lane]);          // g_j / w_j
#pragma unroll 1
        for (int l = 0; l <= D; ++l)
            if (l != lane) term = mont_mul_serial(term, fe_sub(rm, consts[kConstLR + l]));   // * (r - l)
    }
#pragma unroll
    for (int off = 4; off > 0; off >>= 1) term = fe_add(term, shfl_down_fe(term, off));   // lanes 0..7 >= D + 1
    return term;
}

// ---------------------------------------------------------------- constants, transcript init

// Montgomery exponentiation: x^e with x, result in Montgomery form
__device__ __forceinline__ fe mont_pow(const fe &xm, const uint32_t e[8]) {
    fe r = fe_const(1);   // 1 in Montgomery form = R mod p
    for (int i = 255; i >= 0; --i) {
        r = mont_mul(r, r);
        if ((e[i >> 5] >> (i & 31)) & 1u) r = mont_mul(r, xm);
    }
    return r;
}

static __global__ void k_init_consts(fe *c) {
    const int t = threadIdx.x;
    const fe Rm = fe_const(1);
    if (t < 5) {   // l * R
        fe v = fe_zero();
        for (int l = 0; l < t; ++l) v = fe_add(v, Rm);
        c[kConstLR + t] = v;
    }
    // Lagrange weights: thread t -> (D, j) with D = t / 5, j = t % 5
    const int D = t / 5, j = t % 5;
    if (t < 25 && D >= 1 && j <= D) {
        long long w = 1;
        for (int l = 0; l <= D; ++l)
            if (l != j) w *= (j - l);
        const bool neg = w < 0;
        if (neg) w = -w;
        fe wm = fe_zero();                       // |w| * R
        for (long long q = 0; q < w; ++q) wm = fe_add(wm, Rm);
        const uint32_t e[8] = {BZK_P0 - 2, BZK_P1, BZK_P2, BZK_P3, BZK_P4, BZK_P5, BZK_P6, BZK_P7};
        fe inv = mont_pow(wm, e);                // |w|^{-1} * R
        c[kConstInvW + 5 * D + j] = neg ? fe_sub(fe_zero(), inv) : inv;
    } else if (t < 25) {
        c[kConstInvW + t] = fe_zero();
    }
    if (t < 8) {   // 2^(32 t + 64) mod p by doubling
        fe v = fe_zero();
        v.l[0] = 1;
        for (int e = 0; e < 32 * t + 64; ++e) v = fe_add(v, v);
        c[kConstPow2 + t] = v;
    }
}

struct Seed32 { uint8_t b[32]; };

// seeds (device, may be null): per-proof seeds [nproofs][32] (BZK_F_SEEDS_DEVICE), else `seed` for all
static __global__ void k_transcript_init(ProofState *ps, uint32_t nproofs, Seed32 seed, const uint8_t *seeds,
                                         uint64_t first_index, uint32_t k, uint32_t d, uint32_t order) {
    uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= nproofs) return;
    uint32_t st[8];
    if (seeds) {
        Seed32 own;
        for (int i = 0; i < 32; ++i) own.b[i] = seeds[(size_t)b * 32 + i];
        transcript_init(st, own.b, first_index + b, k, d, order);
    } else {
        transcript_init(st, seed.b, first_index + b, k, d, order);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) ps[b].st[i] = st[i];
}

// ---------------------------------------------------------------- global round kernel

// Raw entries of one table for pair j: E = 2 (round 1: a, b) or 4 (fused round: the two fold
// pairs whose results are this round's (a, b)), in the order fold_group consumes them.
template <int ORDER, bool FIRST> struct Geo {
    static constexpr int E = FIRST ? 2 : 4;
};

// element offsets (relative to T + j) of the E raw entries of pair j in a table of E h entries
template <int ORDER, bool FIRST>
__device__ __forceinline__ uint64_t raw_off(uint64_t h, uint64_t j, int e) {
    if (ORDER == 0) return (FIRST ? 2 : 4) * j + e;
    if (FIRST) return j + (e ? h : 0);
    // MSB fused: previous round paired (x, x + 2h); this round pairs (j, j + h)
    return j + (e == 0 ? 0 : e == 1 ? 2 * h : e == 2 ? h : 3 * h);
}

// From the raw entries x[] of table m: round 1 -> (a, b); fused round -> fold both pairs with
// r_{i-1}, store the folded pair to the other ping-pong buffer (Fig. 5), return (a, b - a).
// RAWD: the delta only feeds a tensor-core sum (k_fused_tc<2>), where any operand < 2^256 is exact, so
// it stays b + 2p - a < 4p for every table (no lz_red)
template <int D, int ORDER, bool FIRST, bool RAWD = false>
__device__ __forceinline__ void fold_group(const fe (&x)[Geo<ORDER, FIRST>::E], int m, fe *dst, uint64_t h,
                                           uint64_t j, const fe *sK, uint32_t zmask, fe &a, fe &sv) {
    fe lo, hi;
    if (FIRST) {
        lo = x[0];
        hi = x[1];
    } else {
        lo = BZK_FOLD(x[0], x[1]);
        hi = BZK_FOLD(x[2], x[3]);
        fe *U = dst + (size_t)m * (2 * h);
        BZK_ASSERT(j < h);
        if (ORDER == 0) { st_fe(U + 2 * j, lo); st_fe(U + 2 * j + 1, hi); }
        else            { st_fe(U + j, lo);     st_fe(U + j + h, hi); }
    }
    a = lo;
    // round 1: b; fused rounds: delta (for d = 2 the table-0 delta may stay < 4p: it only
    // meets mul_acc, a full 512-bit product < 8p^2)
    sv = FIRST ? hi : ((RAWD || (D == 2 && m == 0)) ? lz_sub(hi, lo) : lz_red(lz_sub(hi, lo)));
}

template <int D, int ORDER, bool FIRST>
__device__ __forceinline__ void load_pair(const fe *src, fe *dst, uint64_t h, uint64_t j, const fe &rm,
                                          const fe *sK, uint32_t zmask, fe (&a)[D], fe (&sv)[D]) {
    constexpr int E = Geo<ORDER, FIRST>::E;
#pragma unroll
    for (int m = 0; m < D; ++m) {
        const fe *T = src + (size_t)m * (E * h);
        fe x[E];
#pragma unroll
        for (int e = 0; e < E; ++e) x[e] = ld_fe_stream(T + raw_off<ORDER, FIRST>(h, j, e));
        fold_group<D, ORDER, FIRST>(x, m, dst, h, j, sK, zmask, a[m], sv[m]);
    }
}

// ---------------------------------------------------------------- TMA staging (k_round<..., TMA>)
//
// Each warp streams its 32 pairs' raw entries of every table into its own shared-memory slot with
// one elected lane issuing cp.async.bulk.tensor copies (TMA, no registers held in flight) completing
// on a per-(warp, table, stage) mbarrier.  The tensor map views the wave's source buffer as rows of
// 128 B (32 x u32) with the 128-byte swizzle, so the lanes' 32-byte entries (row = the lane's 4
// entries for LSB fused rounds) are read back with bank-conflict-free LDS.128.
//   fused rounds: ONE stage per table; the copy of the next grid-stride tile of table m is issued
//     as soon as table m's entries are folded (all lanes past their last use: __syncwarp), so it
//     lands while the rest of this iteration and the next tables compute;
//   round 1: THREE stages (no fold to hide behind and a short iteration): at the top of iteration n
//     tile n + 2 goes into the stage iteration n - 1 consumed.
// Slot = E KiB per (warp, table, stage): LSB E entries of 32 lanes are one box of E * 8 rows; MSB
// reads E segments of 8 rows (the pairs' halves are h entries apart).
template <int ORDER, bool FIRST> struct TmaGeo {
    static constexpr int E = Geo<ORDER, FIRST>::E;
    static constexpr int NSTAGE = FIRST ? 3 : 1;
    static constexpr uint32_t SLOT = E * 1024;
    static constexpr uint32_t BOX_ROWS = ORDER == 0 ? E * 8 : 8;
};

template <int D, bool FIRST>
constexpr size_t tma_smem_bytes() {   // + 1 KiB: the dynamic base is aligned up to 1 KiB in the kernel
    return (size_t)(BZK_RT / 32) * D * TmaGeo<0, FIRST>::NSTAGE * TmaGeo<0, FIRST>::SLOT + 1024;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t dyn_smem_bytes() {
    uint32_t r;
    asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(r));
    return r;
}

__device__ __forceinline__ void mbar_init(uint64_t *bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile("{\n\t.reg .pred P1;\n\t"
                 "BZK_WAIT:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
                 "@!P1 bra BZK_WAIT;\n\t}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_load_rows(void *dst, const CUtensorMap *tm, uint64_t row, uint64_t *bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(smem_u32(dst)), "l"(tm), "r"(0), "r"((int)row), "r"(smem_u32(bar)) : "memory");
}

// lane 0: arm table m's barrier with the slot's bytes and copy the raw entries of pairs j0..j0+31
template <int ORDER, bool FIRST>
__device__ __forceinline__ void tma_issue(const CUtensorMap *tm, uint8_t *slot, uint64_t *bar, uint64_t row0,
                                          uint64_t h, uint64_t j0) {
    using G = TmaGeo<ORDER, FIRST>;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic reads of the slot before the async writes
    mbar_expect_tx(bar, G::SLOT);
    if (ORDER == 0) {
        tma_load_rows(slot, tm, row0 + j0 * G::E / 4, bar);
    } else {
#pragma unroll
        for (int e = 0; e < G::E; ++e) tma_load_rows(slot + e * 1024, tm, row0 + raw_off<ORDER, FIRST>(h, j0, e) / 4, bar);
    }
}

// raw entry e of this lane's pair from a (swizzled) slot
template <int ORDER, bool FIRST>
__device__ __forceinline__ fe tma_entry(const uint8_t *slot, uint32_t lane, int e) {
    uint32_t seg, row, c0;
    if (ORDER == 0) {
        seg = 0;
        if (FIRST) { row = lane >> 1; c0 = 4 * (lane & 1) + 2 * e; }
        else       { row = lane;      c0 = 2 * e; }
    } else {
        seg = e; row = lane >> 2; c0 = 2 * (lane & 3);
    }
    BZK_ASSERT((seg + 1) * 1024 <= TmaGeo<ORDER, FIRST>::SLOT && row < 8 * (ORDER == 0 ? TmaGeo<ORDER, FIRST>::E : 1));
    const uint8_t *base = slot + seg * 1024 + row * 128;
    const uint4 x = *reinterpret_cast<const uint4 *>(base + ((c0 ^ (row & 7)) << 4));
    const uint4 y = *reinterpret_cast<const uint4 *>(base + (((c0 + 1) ^ (row & 7)) << 4));
    fe r;
    r.l[0] = x.x; r.l[1] = x.y; r.l[2] = x.z; r.l[3] = x.w;
    r.l[4] = y.x; r.l[5] = y.y; r.l[6] = y.z; r.l[7] = y.w;
    return r;
}

// End of a global round kernel, every thread of the CTA: the CTA's sums (acc, per thread) are
// reduced; one partial per CTA (or per thread-block cluster, through DSMEM) goes through the
// last-CTA ticket; the proof's last CTA finalises the round (transcript, r_i, outputs, next claim).
template <int D, bool DERIVE>
__device__ __forceinline__ void round_finish(const RoundParams &P, uint32_t b, fe (&acc)[Pts<D, DERIVE>::NV], fe *s_red,
                                             fe *s_clu, int *s_last_p) {
    constexpr int NV = Pts<D, DERIVE>::NV;
    int &s_last = *s_last_p;
    block_reduce<NV>(acc, s_red);
    fe *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    fe *chals = P.challenges + (size_t)b * P.k;
    fe *claim = P.claims ? P.claims + b : nullptr;
    __shared__ fe s_g[D + 1];
    __shared__ fe s_rm;
    if (P.ctas == 1) {
        if (threadIdx.x < 32) {
            if (threadIdx.x == 0)
                finalize_round<D, DERIVE ? 2 : 1>(acc, P.round, P.ps[b], evals, chals, claim, &s_rm, s_g, P.given);
            __syncwarp();
            const fe c = lagrange_warp<D>(s_g, s_rm, P.consts);
            if (threadIdx.x == 0) P.ps[b].claim = c;
        }
        return;
    }
    // Thread-block cluster (launched with cluster dims (cs, 1, 1), cs <= 8, all CTAs of one proof):
    // the cluster's CTA sums are combined through distributed shared memory, so only one partial
    // per cluster goes to global memory and through the last-CTA ticket.
    namespace cg = cooperative_groups;
    cg::cluster_group cluster = cg::this_cluster();
    const uint32_t cs = cluster.num_blocks();
    if (cs > 1) {
        if (threadIdx.x == 0)
#pragma unroll
            for (int t = 0; t < NV; ++t) s_clu[t] = acc[t];
        cluster.sync();
        const bool leader = cluster.block_rank() == 0;
        if (leader && threadIdx.x == 0) {
            for (uint32_t r = 1; r < cs; ++r) {
                const fe *rem = cluster.map_shared_rank(s_clu, r);
#pragma unroll
                for (int t = 0; t < NV; ++t) acc[t] = fe_add(acc[t], rem[t]);
            }
        }
        cluster.sync();   // remote shared memory must outlive the leader's reads
        if (!leader) return;
    }
    const uint32_t nparts = P.ctas / cs, pidx = blockIdx.x / cs;
    BZK_ASSERT(pidx < nparts && blockIdx.x < P.ctas);
    fe *part = P.partials + (size_t)b * P.ctas * NV;
    if (threadIdx.x == 0) {
#pragma unroll
        for (int t = 0; t < NV; ++t) st_fe_cg(&part[(size_t)pidx * NV + t], acc[t]);
        __threadfence();
        uint32_t old = atomicAdd(&P.tickets[b], 1u);
        s_last = (old == nparts - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // last CTA of proof b: cooperative sum of all partials
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = fe_zero();
    for (uint32_t c = threadIdx.x; c < nparts; c += blockDim.x)
#pragma unroll
        for (int t = 0; t < NV; ++t) acc[t] = fe_add(acc[t], ld_fe_cg(&part[(size_t)c * NV + t]));
    block_reduce<NV>(acc, s_red);
    if (threadIdx.x < 32) {
        if (threadIdx.x == 0) {
            P.tickets[b] = 0;
            finalize_round<D, DERIVE ? 2 : 1>(acc, P.round, P.ps[b], evals, chals, claim, &s_rm, s_g, P.given);
        }
        __syncwarp();
        const fe c = lagrange_warp<D>(s_g, s_rm, P.consts);
        if (threadIdx.x == 0) P.ps[b].claim = c;
    }
}

template <int D, int ORDER, bool FIRST, bool TMA>
__global__ void __launch_bounds__(BZK_RT, (D <= 2 ? BZK_ROUND_OCC : 1))
    k_round(RoundParams P, const __grid_constant__ CUtensorMap tmap) {
    constexpr bool DERIVE = !FIRST;
    constexpr int NV = Pts<D, DERIVE>::NV;
    __shared__ fe s_red[32 * NV];
    __shared__ fe s_clu[NV];
    __shared__ int s_last;
    const uint32_t b = blockIdx.y;
    const uint64_t h = 1ull << P.log_h;
    acc9 wacc[NV];
#pragma unroll
    for (int t = 0; t < NV; ++t) wacc[t] = acc9_zero();

    const fe *src = P.src + (size_t)b * D * (FIRST ? 2 * h : 4 * h);
    fe *dst = FIRST ? nullptr : P.dst + (size_t)b * D * (2 * h);
    const fe rm = FIRST ? fe_zero() : P.ps[b].rmont;
    __shared__ __align__(16) fe sK[8];   // fixed-multiplier table of r_{i-1} (fused rounds)
    if (!FIRST) {
        if (threadIdx.x < 8) sK[threadIdx.x] = mont_mul(rm, P.consts[kConstPow2 + threadIdx.x]);   // r 2^(32t+64)
        __syncthreads();
    }
    const uint64_t stride = (uint64_t)P.ctas * blockDim.x;
    const uint32_t lane = threadIdx.x & 31;
    if constexpr (TMA) {
        using G = TmaGeo<ORDER, FIRST>;
        extern __shared__ uint8_t tma_raw[];
        __shared__ __align__(8) uint64_t bars[(BZK_RT / 32) * D * G::NSTAGE];
        uint8_t *tma_base = tma_raw + ((1024 - (smem_u32(tma_raw) & 1023)) & 1023);
        const uint32_t warp = threadIdx.x >> 5;
        uint8_t *wslots = tma_base + (size_t)warp * D * G::NSTAGE * G::SLOT;
        uint64_t *wbars = bars + warp * D * G::NSTAGE;
        if (lane == 0) {
#pragma unroll
            for (int q = 0; q < D * G::NSTAGE; ++q) mbar_init(&wbars[q]);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncwarp();
        const uint64_t row0 = (uint64_t)b * D * (G::E * h / 4);   // this proof's first row (table 0)
        const uint64_t trows = G::E * h / 4;                       // rows per table
        const uint64_t j0 = (uint64_t)blockIdx.x * blockDim.x + warp * 32;
        if (lane == 0)
#pragma unroll
            for (int s = 0; s < (FIRST ? G::NSTAGE - 1 : 1); ++s)
                if (j0 + s * stride < h)
#pragma unroll
                    for (int m = 0; m < D; ++m)
                        tma_issue<ORDER, FIRST>(&tmap, wslots + (s * D + m) * G::SLOT, &wbars[s * D + m],
                                                row0 + m * trows, h, j0 + s * stride);
        acc17 uacc[NV];
#pragma unroll
        for (int t = 0; t < NV; ++t) uacc[t] = acc17_zero();
        uint32_t it = 0;
        for (uint64_t jw = j0; jw < h; jw += stride, ++it) {
            const uint32_t s = G::NSTAGE == 1 ? 0 : it % G::NSTAGE;
            const uint32_t par = G::NSTAGE == 1 ? (it & 1) : ((it / G::NSTAGE) & 1);
            const uint64_t j = jw + lane;
            if (FIRST && lane == 0 && jw + (G::NSTAGE - 1) * stride < h) {
                // the stage of tile it + NSTAGE - 1 was consumed by iteration it - 1 (__syncwarp below)
                const uint32_t sn = (it + G::NSTAGE - 1) % G::NSTAGE;
#pragma unroll
                for (int m = 0; m < D; ++m)
                    tma_issue<ORDER, FIRST>(&tmap, wslots + (sn * D + m) * G::SLOT, &wbars[sn * D + m],
                                            row0 + m * trows, h, jw + (G::NSTAGE - 1) * stride);
            }
            fe a[D], sv[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                uint8_t *slot = wslots + (s * D + m) * G::SLOT;
                mbar_wait(&wbars[s * D + m], par);
                fe x[G::E];
#pragma unroll
                for (int e = 0; e < G::E; ++e) x[e] = tma_entry<ORDER, FIRST>(slot, lane, e);
                fold_group<D, ORDER, FIRST>(x, m, dst, h, j, sK, P.zero, a[m], sv[m]);
                if (!FIRST) {
                    __syncwarp();            // every lane has consumed the slot (the folds used x[])
                    if (lane == 0 && jw + stride < h)
                        tma_issue<ORDER, FIRST>(&tmap, slot, &wbars[m], row0 + m * trows, h, jw + stride);
                }
            }
            if constexpr (D >= 2) {
                eval_one<D, DERIVE>(a, sv, uacc);
            } else {
                acc9_add(wacc[0], a[0]);
                if (!DERIVE) acc9_add(wacc[1], sv[0]);
            }
            if (FIRST) __syncwarp();         // the evaluation consumed every lane's entries of stage s
        }
        if constexpr (D >= 2) {
#pragma unroll
            for (int t = 0; t < NV; ++t) { wacc[t].lo = acc17_to_fe(uacc[t]); wacc[t].hi = 0; }
        }
    } else if constexpr (D >= 2) {
        // One pair per loop iteration; the last product of every point goes unreduced into a
        // 544-bit accumulator, reduced once after the loop.
        acc17 uacc[NV];
#pragma unroll
        for (int t = 0; t < NV; ++t) uacc[t] = acc17_zero();
        for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < h; j += stride) {
            fe a[D], sv[D];
            load_pair<D, ORDER, FIRST>(src, dst, h, j, rm, sK, P.zero, a, sv);
            eval_one<D, DERIVE>(a, sv, uacc);
        }
#pragma unroll
        for (int t = 0; t < NV; ++t) { wacc[t].lo = acc17_to_fe(uacc[t]); wacc[t].hi = 0; }
    } else {
        fe ha[D], hs[D];
        bool held = false;
        for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < h; j += stride) {
            fe a[D], sv[D];
            load_pair<D, ORDER, FIRST>(src, dst, h, j, rm, sK, P.zero, a, sv);
            if (held) {
                eval_two<D, DERIVE>(ha, hs, a, sv, wacc);
            } else {
#pragma unroll
                for (int m = 0; m < D; ++m) { ha[m] = a[m]; hs[m] = sv[m]; }
            }
            held = !held;
        }
        if (held) {
            fe z[D];
#pragma unroll
            for (int m = 0; m < D; ++m) z[m] = fe_zero();
            eval_two<D, DERIVE>(ha, hs, z, z, wacc);
        }
    }

    fe acc[NV];
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = acc9_to_fe(wacc[t]);
    round_finish<D, DERIVE>(P, b, acc, s_red, s_clu, &s_last);
}

// ---------------------------------------------------------------- on-chip tail

struct TailParams {
    const fe *src;        // i0 == 1: [Bw][D][2h0] (input); else [Bw][D][4h0] (unfolded)
    uint32_t log_h0;      // pairs in the first tail round
    uint32_t i0;          // first tail round
    uint32_t k, order;
    ProofState *ps;
    fe *round_evals, *challenges, *final_evals, *claims;
    const fe *consts;
    uint32_t given;       // 1: challenges are inputs (BZK_F_GIVEN_CHALLENGES), no transcript
    uint32_t folded;      // 1: src holds the round-i0 table itself ([D][2h0] per proof, i0 > 1: k_multi)
    uint64_t src_stride;  // elements per proof in src (0: the default D * 2h0 or D * 4h0)
};

template <int D, int ORDER>
__global__ void __launch_bounds__(256) k_tail(TailParams P) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ fe s_red[32 * (D + 1)];
    __shared__ fe s_r;
    const uint32_t b = blockIdx.x;
    const uint32_t h0 = 1u << P.log_h0;
    fe *A = reinterpret_cast<fe *>(smem_raw);          // [D][2h0]
    fe *Bf = A + (size_t)D * 2 * h0;                   // [D][h0]
    fe *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    fe *chals = P.challenges + (size_t)b * P.k;
    fe *claim = P.claims ? P.claims + b : nullptr;

    if (P.k == 0) {  // no rounds: final_m = T_m[0], claim = prod_m T_m[0]
        if (threadIdx.x == 0) {
            const fe *src = P.src + (size_t)b * D;
            fe prod = ld_fe(src);
            st_fe(&P.final_evals[(size_t)b * D], prod);
            for (int m = 1; m < D; ++m) {
                fe v = ld_fe(src + m);
                st_fe(&P.final_evals[(size_t)b * D + m], v);
                prod = mont_mul(prod, v);
            }
            if (claim) st_fe(claim, mont_mul(prod, fe_R_pow(D)));
        }
        return;
    }

    // stage the round-i0 table (2h0 entries per m) into A.  Tables 1..D-1 are held in Montgomery
    // form (x R): a product v_0 v_1 ... v_{D-1} through D-1 Montgomery products then comes out in
    // standard form (no per-round R^{-(D-1)} fix on the serial path); folds are linear, so the form is
    // kept; the final evaluations are converted back.
    const fe R2 = fe_const(2);
    if (P.i0 == 1 || P.folded) {
        const fe *src = P.src + (size_t)b * (P.src_stride ? P.src_stride : (size_t)D * (2 * h0));
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) {
            const fe v = ld_fe(src + x);
            A[x] = x < 2 * h0 ? v : mont_mul(v, R2);
        }
    } else {
        const fe *src = P.src + (size_t)b * D * (4 * h0);
        const fe rm = P.ps[b].rmont;
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) {
            uint32_t m = x / (2 * h0), y = x % (2 * h0);
            const fe *T = src + (size_t)m * 4 * h0;
            fe lo, hi;
            if (ORDER == 0) { lo = ld_fe(T + 2 * y); hi = ld_fe(T + 2 * y + 1); }
            else            { lo = ld_fe(T + y);     hi = ld_fe(T + y + 2 * h0); }
            // entries written by a fused round are lazily reduced (< 2p): canonicalise first
            const fe v = fold1(fe_reduce_once(lo), fe_reduce_once(hi), rm);
            A[x] = m == 0 ? v : mont_mul(v, R2);
        }
    }
    __syncthreads();

    fe *cur = A, *oth = Bf;
    uint32_t h = h0;
    for (uint32_t i = P.i0; i <= P.k; ++i) {
        fe acc[D + 1];
#pragma unroll
        for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
        for (uint32_t j = threadIdx.x; j < h; j += blockDim.x) {
            fe a[D], bb[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const fe *T = cur + (size_t)m * 2 * h;
                if (ORDER == 0) { a[m] = T[2 * j]; bb[m] = T[2 * j + 1]; }
                else            { a[m] = T[j];     bb[m] = T[j + h]; }
            }
            eval_pair<D>(a, bb, acc);
        }
        block_reduce<D + 1>(acc, s_red);
        if (threadIdx.x == 0) {
            fe rm;
            finalize_round<D, 0>(acc, i, P.ps[b], evals, chals, claim, &rm, nullptr, P.given);
            s_r = rm;
        }
        __syncthreads();
        const fe rm = s_r;
        // fold cur (2h per m) -> oth (h per m)
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * h; x += blockDim.x) {
            uint32_t m = x / h, j = x % h;
            const fe *T = cur + (size_t)m * 2 * h;
            fe lo, hi;
            if (ORDER == 0) { lo = T[2 * j]; hi = T[2 * j + 1]; }
            else            { lo = T[j];     hi = T[j + h]; }
            oth[(size_t)m * h + j] = fold1(lo, hi, rm);
        }
        __syncthreads();
        fe *tmp = cur; cur = oth; oth = tmp;
        h >>= 1;
    }
    // after round k the tables have one entry: final_m = f_m(rho) (tables 1..D-1 back from Montgomery form)
    if (threadIdx.x < D) {
        fe one = fe_zero();
        one.l[0] = 1;
        const fe v = cur[threadIdx.x];
        st_fe(&P.final_evals[(size_t)b * D + threadIdx.x], threadIdx.x == 0 ? v : mont_mul(v, one));
    }
}

// launchers, explicitly instantiated per degree in k_d<D>.cu (parallel compilation)
template <int D>
cudaError_t launch_round(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                         const RoundParams &p, const CUtensorMap &tm);
template <int D>
cudaError_t launch_tail(uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                        const TailParams &p);
template <int D>
cudaError_t set_kernel_attrs();   // once per process, before any launch or graph capture
// k_round1_tc (round1_tc.cuh, k_r1tc.cu): d = 2 round 1 on the tensor cores
cudaError_t r1tc_launch(uint32_t order, bool sw64, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm);
cudaError_t r1tc_set_attrs();   // and k_fused_tc's
// k_fused_tc (fused_tc.cuh, k_r1tc.cu): d = 2 fused rounds, d = 3 round 1 and fused rounds with the
// evaluation sums on the tensor cores
// (small: the NW = 2 variant of the d = 2 fused rounds, api.cu ftc_small)
cudaError_t ftc_launch(uint32_t D, bool first, bool small, uint32_t order, dim3 grid, cudaStream_t s,
                       const RoundParams &p, const CUtensorMap &tm);

}  // namespace bzk
