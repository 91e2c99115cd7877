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
//       Each thread takes two pairs at a time and sums their products with ONE Montgomery
//       reduction (mont_mul2).  Partial sums: per thread -> warp shuffle -> shared memory ->
//       per-CTA partial in global -> last-CTA ticket; the last CTA of each proof reduces the
//       partials, hashes the transcript and publishes r_i (single pass, no extra launch; the
//       paper's reduction made repeated global passes).
//   k_tail<D,ORDER>  one CTA per proof finishes the remaining rounds (h <= tail threshold) in
//       shared memory, including the final fold that yields final_m = f_m(rho).
#pragma once
#include <stdint.h>
#include "field.cuh"

#ifndef BZK_ROUND_OCC
#define BZK_ROUND_OCC 2   // resident CTAs per SM requested for k_round (d <= 2)
#endif
#include "sha256.cuh"

namespace bzk {

struct ProofState {
    uint32_t st[8];   // transcript state_i
    fe rmont;         // r_i * R mod p (Montgomery) for the next fold
    fe claim;         // claim_{i+1} = g_i(r_i) (standard form)
};

// Device constants (filled once per context by k_init_consts):
//   [0..4]        l * R mod p, l = 0..4          (Montgomery form of the node l)
//   [5 + 5D + j]  w_{D,j}^{-1} * R mod p, w_{D,j} = prod_{l != j, 0<=l<=D} (j - l)   (Lagrange)
constexpr int kConstLR = 0;
constexpr int kConstInvW = 5;
constexpr int kNumConsts = 5 + 5 * 5;

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
    uint32_t prefetch;    // 1: bulk-prefetch the next iteration's tiles into L2
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

// number of summed evaluation points: all t = 0..D, or t in {0, 2..D} when g(1) is derived
template <int D, bool DERIVE> struct Pts { static constexpr int NV = DERIVE ? D : D + 1; };

// Evaluate two pairs (a, a + delta) and (a2, a2 + delta2) at the summed points and accumulate.
// a / a2 are overwritten (they walk through v(t) = a + t*delta).  Products of the two pairs
// share one Montgomery reduction (mont_mul2); every sum carries R^{-(D-1)}.
template <int D, bool DERIVE>
__device__ __forceinline__ void eval_two(fe (&a)[D], const fe (&delta)[D], fe (&a2)[D], const fe (&delta2)[D],
                                         fe (&acc)[Pts<D, DERIVE>::NV]) {
#pragma unroll
    for (int t = 0; t <= D; ++t) {
        if (t > 0) {
#pragma unroll
            for (int m = 0; m < D; ++m) { a[m] = fe_add(a[m], delta[m]); a2[m] = fe_add(a2[m], delta2[m]); }
        }
        if (DERIVE && t == 1) continue;
        const int idx = DERIVE ? (t == 0 ? 0 : t - 1) : t;
        if (D == 1) {
            acc[idx] = fe_add(acc[idx], fe_add(a[0], a2[0]));
        } else {
            fe p = a[0], p2 = a2[0];
#pragma unroll
            for (int m = 1; m < D - 1; ++m) { p = mont_mul(p, a[m]); p2 = mont_mul(p2, a2[m]); }
            acc[idx] = fe_add(acc[idx], mont_mul2(p, a[D - 1], p2, a2[D - 1]));
        }
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

// ---------------------------------------------------------------- per-round finalisation

// g(r) from g(0..D) by Lagrange interpolation on the nodes 0..D (all standard form; rm = r R).
template <int D>
__device__ __forceinline__ fe lagrange_at(const fe (&g)[D + 1], const fe &rm, const fe *consts) {
    fe acc = fe_zero();
#pragma unroll 1
    for (int j = 0; j <= D; ++j) {
        fe term = mont_mul(g[j], consts[kConstInvW + 5 * D + j]);          // g_j / w_j
#pragma unroll 1
        for (int l = 0; l <= D; ++l)
            if (l != j) term = mont_mul(term, fe_sub(rm, consts[kConstLR + l]));   // * (r - l)
        acc = fe_add(acc, term);
    }
    return acc;
}

// Fix the R^{-(D-1)} scale of the round sums, complete g(1) when derived, absorb g into the
// transcript, derive r_i, write the round's outputs and the next claim.  ONE thread per proof.
template <int D, bool DERIVE>
__device__ __forceinline__ void finalize_round(fe (&S)[Pts<D, DERIVE>::NV], uint32_t round, ProofState &ps,
                                               fe *round_evals, fe *challenges, fe *claims, const fe *consts,
                                               fe *rmont_out) {
    fe g[D + 1];
    const fe RD = fe_R_pow(D);
    if (DERIVE) {
        g[0] = mont_mul(S[0], RD);
        g[1] = fe_sub(ps.claim, g[0]);
#pragma unroll
        for (int t = 2; t <= D; ++t) g[t] = mont_mul(S[t - 1], RD);
    } else {
#pragma unroll
        for (int t = 0; t <= D; ++t) g[t] = mont_mul(S[t], RD);
    }
    uint32_t st[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) st[i] = ps.st[i];
    fe r = transcript_round(st, g, D);
#pragma unroll
    for (int i = 0; i < 8; ++i) ps.st[i] = st[i];
#pragma unroll
    for (int t = 0; t <= D; ++t) st_fe(&round_evals[(size_t)(round - 1) * (D + 1) + t], g[t]);
    st_fe(&challenges[round - 1], r);
    if (round == 1 && claims) st_fe(claims, fe_add(g[0], g[1]));
    fe rm = mont_mul(r, fe_const(2));
    ps.rmont = rm;
    ps.claim = lagrange_at<D>(g, rm, consts);
    if (rmont_out) *rmont_out = rm;
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
}

struct Seed32 { uint8_t b[32]; };

static __global__ void k_transcript_init(ProofState *ps, uint32_t nproofs, Seed32 seed, uint64_t first_index,
                                         uint32_t k, uint32_t d, uint32_t order) {
    uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= nproofs) return;
    uint32_t st[8];
    transcript_init(st, seed.b, first_index + b, k, d, order);
#pragma unroll
    for (int i = 0; i < 8; ++i) ps[b].st[i] = st[i];
}

// ---------------------------------------------------------------- global round kernel

template <int D, int ORDER, bool FIRST>
__device__ __forceinline__ void load_pair(const fe *src, fe *dst, uint64_t h, uint64_t j, const fe &rm,
                                          fe (&a)[D], fe (&delta)[D]) {
#pragma unroll
    for (int m = 0; m < D; ++m) {
        fe lo, hi;
        if (FIRST) {
            const fe *T = src + (size_t)m * (2 * h);
            if (ORDER == 0) { lo = ld_fe_stream(T + 2 * j); hi = ld_fe_stream(T + 2 * j + 1); }
            else            { lo = ld_fe_stream(T + j);     hi = ld_fe_stream(T + j + h); }
        } else {
            const fe *T = src + (size_t)m * (4 * h);
            fe *U = dst + (size_t)m * (2 * h);
            if (ORDER == 0) {
                fe x0 = ld_fe_stream(T + 4 * j), x1 = ld_fe_stream(T + 4 * j + 1);
                fe x2 = ld_fe_stream(T + 4 * j + 2), x3 = ld_fe_stream(T + 4 * j + 3);
                lo = fold1(x0, x1, rm);
                hi = fold1(x2, x3, rm);
                st_fe(U + 2 * j, lo);
                st_fe(U + 2 * j + 1, hi);
            } else {
                // previous round paired (x, x + 2h); this round pairs (j, j + h)
                fe x0 = ld_fe_stream(T + j), x1 = ld_fe_stream(T + j + 2 * h);
                fe x2 = ld_fe_stream(T + j + h), x3 = ld_fe_stream(T + j + 3 * h);
                lo = fold1(x0, x1, rm);
                hi = fold1(x2, x3, rm);
                st_fe(U + j, lo);
                st_fe(U + j + h, hi);
            }
        }
        a[m] = lo;
        delta[m] = fe_sub(hi, lo);
    }
}

// L2 bulk prefetch of a contiguous byte range (cp.async.bulk.prefetch, sm_90+; no registers, no smem)
__device__ __forceinline__ void prefetch_l2(const void *p, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// Lane 0 of a warp prefetches into L2 the table ranges that the warp's 32 lanes will load for the
// pairs j0 .. j0+31 (j0 = the warp's first pair index): one contiguous range per table for LSB,
// two for MSB.
template <int D, int ORDER, bool FIRST>
__device__ __forceinline__ void prefetch_pairs(const fe *src, uint64_t h, uint64_t j0) {
    if (j0 >= h) return;
    const uint64_t n = (h - j0) < 32 ? (h - j0) : 32;
#pragma unroll
    for (int m = 0; m < D; ++m) {
        if (FIRST) {
            const fe *T = src + (size_t)m * (2 * h);
            if (ORDER == 0) prefetch_l2(T + 2 * j0, (uint32_t)(n * 64));
            else { prefetch_l2(T + j0, (uint32_t)(n * 32)); prefetch_l2(T + j0 + h, (uint32_t)(n * 32)); }
        } else {
            const fe *T = src + (size_t)m * (4 * h);
            if (ORDER == 0) prefetch_l2(T + 4 * j0, (uint32_t)(n * 128));
            else {
                prefetch_l2(T + j0, (uint32_t)(n * 32));
                prefetch_l2(T + j0 + h, (uint32_t)(n * 32));
                prefetch_l2(T + j0 + 2 * h, (uint32_t)(n * 32));
                prefetch_l2(T + j0 + 3 * h, (uint32_t)(n * 32));
            }
        }
    }
}

template <int D, int ORDER, bool FIRST>
__global__ void __launch_bounds__(256, (D <= 2 ? BZK_ROUND_OCC : 1)) k_round(RoundParams P) {
    constexpr bool DERIVE = !FIRST;
    constexpr int NV = Pts<D, DERIVE>::NV;
    __shared__ fe s_red[32 * NV];
    __shared__ int s_last;
    const uint32_t b = blockIdx.y;
    const uint64_t h = 1ull << P.log_h;
    fe acc[NV];
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = fe_zero();

    const fe *src = P.src + (size_t)b * D * (FIRST ? 2 * h : 4 * h);
    fe *dst = FIRST ? nullptr : P.dst + (size_t)b * D * (2 * h);
    const fe rm = FIRST ? fe_zero() : P.ps[b].rmont;
    const uint64_t stride = (uint64_t)P.ctas * blockDim.x;
    const uint32_t lane = threadIdx.x & 31;
    for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < h; j += 2 * stride) {
        if (P.prefetch && lane == 0) {
            prefetch_pairs<D, ORDER, FIRST>(src, h, j + 2 * stride);
            prefetch_pairs<D, ORDER, FIRST>(src, h, j + 3 * stride);
        }
        fe a[D], da[D], a2[D], da2[D];
        load_pair<D, ORDER, FIRST>(src, dst, h, j, rm, a, da);
        const uint64_t j2 = j + stride;
        if (j2 < h) {
            load_pair<D, ORDER, FIRST>(src, dst, h, j2, rm, a2, da2);
        } else {
#pragma unroll
            for (int m = 0; m < D; ++m) { a2[m] = fe_zero(); da2[m] = fe_zero(); }
        }
        eval_two<D, DERIVE>(a, da, a2, da2, acc);
    }

    block_reduce<NV>(acc, s_red);
    fe *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    fe *chals = P.challenges + (size_t)b * P.k;
    fe *claim = P.claims ? P.claims + b : nullptr;
    if (P.ctas == 1) {
        if (threadIdx.x == 0)
            finalize_round<D, DERIVE>(acc, P.round, P.ps[b], evals, chals, claim, P.consts, nullptr);
        return;
    }
    fe *part = P.partials + (size_t)b * P.ctas * NV;
    if (threadIdx.x == 0) {
#pragma unroll
        for (int t = 0; t < NV; ++t) st_fe_cg(&part[(size_t)blockIdx.x * NV + t], acc[t]);
        __threadfence();
        uint32_t old = atomicAdd(&P.tickets[b], 1u);
        s_last = (old == P.ctas - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // last CTA of proof b: cooperative sum of all partials
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = fe_zero();
    for (uint32_t c = threadIdx.x; c < P.ctas; c += blockDim.x)
#pragma unroll
        for (int t = 0; t < NV; ++t) acc[t] = fe_add(acc[t], ld_fe_cg(&part[(size_t)c * NV + t]));
    block_reduce<NV>(acc, s_red);
    if (threadIdx.x == 0) {
        P.tickets[b] = 0;
        finalize_round<D, DERIVE>(acc, P.round, P.ps[b], evals, chals, claim, P.consts, nullptr);
    }
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

    // stage the round-i0 table (2h0 entries per m) into A
    if (P.i0 == 1) {
        const fe *src = P.src + (size_t)b * D * (2 * h0);
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) A[x] = ld_fe(src + x);
    } else {
        const fe *src = P.src + (size_t)b * D * (4 * h0);
        const fe rm = P.ps[b].rmont;
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) {
            uint32_t m = x / (2 * h0), y = x % (2 * h0);
            const fe *T = src + (size_t)m * 4 * h0;
            fe lo, hi;
            if (ORDER == 0) { lo = ld_fe(T + 2 * y); hi = ld_fe(T + 2 * y + 1); }
            else            { lo = ld_fe(T + y);     hi = ld_fe(T + y + 2 * h0); }
            A[x] = fold1(lo, hi, rm);
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
            finalize_round<D, false>(acc, i, P.ps[b], evals, chals, claim, P.consts, &rm);
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
    // after round k the tables have one entry: final_m = f_m(rho)
    if (threadIdx.x < D) st_fe(&P.final_evals[(size_t)b * D + threadIdx.x], cur[threadIdx.x]);
}

// launchers, explicitly instantiated per degree in k_d<D>.cu (parallel compilation)
template <int D>
cudaError_t launch_round(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                         const RoundParams &p);
template <int D>
cudaError_t launch_tail(uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                        const TailParams &p);
template <int D>
cudaError_t set_kernel_attrs();   // once per process, before any launch or graph capture

}  // namespace bzk
