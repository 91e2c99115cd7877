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
//       FIRST : round 1, evaluation only (reads the input once).
//       !FIRST: fused fold(r_{i-1}) + eval(i): a thread reads 4 entries per table, writes the 2
//               folded ones to the other ping-pong buffer (Fig. 5) and evaluates round i
//               on them in registers (the sums reuse the update's loads).
//       Partial sums: per thread -> warp shuffle -> shared memory -> per-CTA partial in global ->
//       last-CTA ticket; the last CTA of each proof reduces the partials, hashes the transcript
//       and publishes r_i (single pass, no extra launch; P:167 did repeated global passes).
//   k_tail<D,ORDER>  one CTA per proof finishes the remaining rounds (h <= tail threshold) in
//       shared memory, including the final fold that yields final_m = f_m(rho).
#pragma once
#include <stdint.h>
#include "field.cuh"
#include "sha256.cuh"

namespace bzk {

struct ProofState {
    uint32_t st[8];   // transcript state_{i}
    fe rmont;         // r_i * R mod p (Montgomery) for the next fold
};

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
    const uint8_t *seed;  // 32 B (device)
    uint64_t first_index;
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

// Fix the R^{-(D-1)} scale of the round sums, absorb them into the transcript, derive r_i and
// write the round's outputs.  Called by ONE thread per proof.
template <int D>
__device__ __forceinline__ void finalize_round(fe (&S)[D + 1], uint32_t round, uint32_t k,
                                               ProofState &ps, fe *round_evals, fe *challenges,
                                               fe *claims, fe *rmont_out) {
    fe g[D + 1];
    const fe RD = fe_R_pow(D);
#pragma unroll
    for (int t = 0; t <= D; ++t) g[t] = mont_mul(S[t], RD);
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
    if (rmont_out) *rmont_out = rm;
}

// ---------------------------------------------------------------- transcript init

static __global__ void k_transcript_init(ProofState *ps, uint32_t nproofs, const uint8_t *seed,
                                  uint64_t first_index, uint32_t k, uint32_t d, uint32_t order) {
    uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= nproofs) return;
    uint8_t s[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) s[i] = seed[i];
    uint32_t st[8];
    transcript_init(st, s, first_index + b, k, d, order);
#pragma unroll
    for (int i = 0; i < 8; ++i) ps[b].st[i] = st[i];
}

// ---------------------------------------------------------------- global round kernel

template <int D, int ORDER, bool FIRST>
__global__ void __launch_bounds__(256, (D <= 2 ? 2 : 1)) k_round(RoundParams P) {
    __shared__ fe s_red[32 * (D + 1)];
    __shared__ int s_last;
    const uint32_t b = blockIdx.y;
    const uint64_t h = 1ull << P.log_h;
    fe acc[D + 1];
#pragma unroll
    for (int t = 0; t <= D; ++t) acc[t] = fe_zero();

    const uint64_t stride = (uint64_t)P.ctas * blockDim.x;
    if (FIRST) {
        const fe *src = P.src + (size_t)b * D * (2 * h);
        for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < h; j += stride) {
            fe a[D], bb[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const fe *T = src + (size_t)m * (2 * h);
                if (ORDER == 0) { a[m] = ld_fe_stream(T + 2 * j); bb[m] = ld_fe_stream(T + 2 * j + 1); }
                else            { a[m] = ld_fe_stream(T + j);     bb[m] = ld_fe_stream(T + j + h); }
            }
            eval_pair<D>(a, bb, acc);
        }
    } else {
        const fe *src = P.src + (size_t)b * D * (4 * h);
        fe *dst = P.dst + (size_t)b * D * (2 * h);
        const fe rm = P.ps[b].rmont;
        for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < h; j += stride) {
            fe a[D], bb[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const fe *T = src + (size_t)m * (4 * h);
                fe *U = dst + (size_t)m * (2 * h);
                if (ORDER == 0) {
                    fe x0 = ld_fe_stream(T + 4 * j), x1 = ld_fe_stream(T + 4 * j + 1);
                    fe x2 = ld_fe_stream(T + 4 * j + 2), x3 = ld_fe_stream(T + 4 * j + 3);
                    a[m] = fold1(x0, x1, rm);
                    bb[m] = fold1(x2, x3, rm);
                    st_fe(U + 2 * j, a[m]);
                    st_fe(U + 2 * j + 1, bb[m]);
                } else {
                    // previous round paired (x, x + 2h); this round pairs (j, j + h)
                    fe x0 = ld_fe_stream(T + j), x1 = ld_fe_stream(T + j + 2 * h);
                    fe x2 = ld_fe_stream(T + j + h), x3 = ld_fe_stream(T + j + 3 * h);
                    a[m] = fold1(x0, x1, rm);
                    bb[m] = fold1(x2, x3, rm);
                    st_fe(U + j, a[m]);
                    st_fe(U + j + h, bb[m]);
                }
            }
            eval_pair<D>(a, bb, acc);
        }
    }

    block_reduce<D + 1>(acc, s_red);
    fe *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    fe *chals = P.challenges + (size_t)b * P.k;
    fe *claim = P.claims ? P.claims + b : nullptr;
    if (P.ctas == 1) {
        if (threadIdx.x == 0) finalize_round<D>(acc, P.round, P.k, P.ps[b], evals, chals, claim, nullptr);
        return;
    }
    fe *part = P.partials + (size_t)b * P.ctas * (D + 1);
    if (threadIdx.x == 0) {
#pragma unroll
        for (int t = 0; t <= D; ++t) st_fe_cg(&part[(size_t)blockIdx.x * (D + 1) + t], acc[t]);
        __threadfence();
        uint32_t old = atomicAdd(&P.tickets[b], 1u);
        s_last = (old == P.ctas - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // last CTA of proof b: cooperative sum of all partials
#pragma unroll
    for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
    for (uint32_t c = threadIdx.x; c < P.ctas; c += blockDim.x)
#pragma unroll
        for (int t = 0; t <= D; ++t) acc[t] = fe_add(acc[t], ld_fe_cg(&part[(size_t)c * (D + 1) + t]));
    block_reduce<D + 1>(acc, s_red);
    if (threadIdx.x == 0) {
        P.tickets[b] = 0;
        finalize_round<D>(acc, P.round, P.k, P.ps[b], evals, chals, claim, nullptr);
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
            finalize_round<D>(acc, i, P.k, P.ps[b], evals, chals, claim, &rm);
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

}  // namespace bzk
