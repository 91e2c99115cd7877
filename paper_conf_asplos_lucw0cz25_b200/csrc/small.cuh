// small.cuh -- one persistent launch per batch for proofs whose tables fit in a thread-block
// cluster's shared memory (cluster/DSMEM reduction, the persistent
// per-proof kernel).
//
// A proof is owned by a cluster of CS = 2^c CTAs (c <= 3).  Its d tables (2^k entries each) are split
// so that every pair of the first k - c rounds is CTA-local:
//   LSB (pairs 2j, 2j+1; north star):   CTA q holds the contiguous slice x in [q 2^(k-c), (q+1) 2^(k-c))
//   MSB (pairs j, j+h; Alg. 1):   CTA q holds the residue class x = q (mod CS), at x / CS
// Folding keeps both layouts CTA-local (LSB: 2j, 2j+1 -> j stays in the slice; MSB: h is a multiple
// of CS, so j and j + h share the residue), so a round is: local evaluation (all points t = 0..d) ->
// block reduction -> partial in shared memory -> cluster barrier -> the leader CTA sums the CS
// per-warp partials over DSMEM, hashes the transcript (SHA-256) and publishes r_i R in its shared
// memory -> cluster barrier -> every CTA reads r_i over DSMEM and folds locally (P:111 line 5).  The
// last c rounds run in the leader on the CS remaining entries per table it gathers over DSMEM.
// Tables 1..d-1 are held in Montgomery form (products come out in standard form, no per-round scale
// fix).  One launch covers every round of every proof of the batch: no per-round kernel boundary, no
// HBM round trip of the folded tables -- the B200 form of the paper's "one proof per cycle" pipeline
// for small batches, where the per-round global kernels are latency-bound.
#pragma once
#include <cooperative_groups.h>
#include <stdint.h>
#include "field.cuh"
#include "sumcheck.cuh"

namespace bzk {

struct SmallParams {
    const fe *src;          // [B][D][2^k] (canonical, standard form)
    uint32_t k, cs_log;     // CS = 2^cs_log CTAs per proof (cluster x-dimension)
    uint32_t order, given;
    uint64_t first_index;
    Seed32 seed;            // transcript seed (or per-proof device seeds)
    const uint8_t *seeds;   // BZK_F_SEEDS_DEVICE: [B][32], else null
    ProofState *ps;         // [B]
    fe *round_evals, *challenges, *final_evals, *claims;
};

template <int D>
constexpr size_t small_smem_bytes(uint32_t nl) { return (size_t)D * nl * 3 / 2 * sizeof(fe); }

template <int D, int ORDER>
__global__ void __launch_bounds__(256) k_small(SmallParams P) {
    namespace cg = cooperative_groups;
    cg::cluster_group cl = cg::this_cluster();
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ fe s_wpart[8][D + 1];      // this CTA's per-warp round partials
    __shared__ fe s_cpart[D + 1];         // this CTA's round partial (the leader reads it over DSMEM)
    __shared__ fe s_rm;                   // leader: r_i R for every CTA of the cluster
    __shared__ fe s_g[2][D][8];           // leader: the last c rounds on the gathered entries
    const uint32_t CS = 1u << P.cs_log, q = cl.block_rank();
    const uint32_t b = blockIdx.y;
    const uint32_t k = P.k;
    uint32_t nl = 1u << (k - P.cs_log);   // local entries per table
    fe *cur = reinterpret_cast<fe *>(smem_raw);    // [D][nl]
    fe *oth = cur + (size_t)D * nl;                  // [D][nl / 2]
    fe *evals = P.round_evals + (size_t)b * k * (D + 1);
    fe *chals = P.challenges + (size_t)b * k;
    fe *claim = P.claims ? P.claims + b : nullptr;
    // the transcript state lives in the leader's shared memory for the whole proof (the per-round
    // finalisation is the serial critical path: no global-memory round trip for state_i)
    __shared__ ProofState s_ps;
    ProofState &ps = s_ps;

    if (q == 0 && threadIdx.x == 0 && !P.given) {    // state_0 (P:211 seed; reading R6)
        uint32_t st[8];
        if (P.seeds) {
            Seed32 own;
            for (int i = 0; i < 32; ++i) own.b[i] = P.seeds[(size_t)b * 32 + i];
            transcript_init(st, own.b, P.first_index + b, k, D, ORDER);
        } else {
            transcript_init(st, P.seed.b, P.first_index + b, k, D, ORDER);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) ps.st[i] = st[i];
    }
    // load this CTA's share (tables 1..D-1 to Montgomery form)
    const fe *src = P.src + (size_t)b * D * ((size_t)1 << k);
    const fe R2 = fe_const(2);
    for (uint32_t x = threadIdx.x; x < (uint32_t)D * nl; x += blockDim.x) {
        const uint32_t m = x / nl, xl = x % nl;
        const uint64_t gx = ORDER == 0 ? (uint64_t)q * nl + xl : (uint64_t)xl * CS + q;
        const fe v = ld_fe(src + (size_t)m * ((size_t)1 << k) + gx);
        cur[x] = m == 0 ? v : mont_mul(v, R2);
    }
    __syncthreads();

    // round 1's evaluation on the loaded table; afterwards every pass folds with r_i AND evaluates
    // round i + 1 on the folded entries (4 reads, 2 writes per next-round pair, as the global fused
    // kernel), so a round is one pass over shared memory
    auto eval_round = [&](fe (&acc)[D + 1], uint32_t n) {
        const uint32_t h = n / 2;
        for (uint32_t j = threadIdx.x; j < h; j += blockDim.x) {
            fe a[D], bb[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const fe *T = cur + (size_t)m * n;
                if (ORDER == 0) { a[m] = T[2 * j]; bb[m] = T[2 * j + 1]; }
                else            { a[m] = T[j];     bb[m] = T[j + h]; }
            }
            eval_pair<D>(a, bb, acc);
        }
    };
    fe acc[D + 1];
#pragma unroll
    for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
    if (nl >= 2) eval_round(acc, nl);
    uint32_t round = 1;
    for (; nl >= 2; ++round) {
        // warp sums -> shared memory -> the CTA's partial (warp 0, lanes 0..7: local loads, 3-level
        // shuffle tree); after the cluster barrier the leader warp's lanes 0..CS-1 each load ONE remote
        // CTA partial and a 3-level shuffle tree sums them (phase trace: the previous one-warp gather of
        // all 8 CS warp partials took 3.8 K cycles per round, profiles/r02/r02k_trace_small_c1.txt)
        warp_reduce<D + 1>(acc);
        const uint32_t lane = threadIdx.x & 31;
        if (lane == 0)
#pragma unroll
            for (int t = 0; t <= D; ++t) s_wpart[threadIdx.x >> 5][t] = acc[t];
        __syncthreads();
        if (threadIdx.x < 32) {
#pragma unroll
            for (int t = 0; t <= D; ++t) acc[t] = lane < 8 ? s_wpart[lane][t] : fe_zero();
#pragma unroll
            for (int off = 4; off > 0; off >>= 1)
#pragma unroll
                for (int t = 0; t <= D; ++t) acc[t] = fe_add(acc[t], shfl_down_fe(acc[t], off));
            if (lane == 0)
#pragma unroll
                for (int t = 0; t <= D; ++t) s_cpart[t] = acc[t];
        }
        cl.sync();                                    // CTA partials visible cluster-wide
        if (q == 0 && threadIdx.x < 32) {
#pragma unroll
            for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
            if (lane < CS) {
                const fe *rp = cl.map_shared_rank(s_cpart, lane);
#pragma unroll
                for (int t = 0; t <= D; ++t) acc[t] = rp[t];
            }
#pragma unroll
            for (int off = 4; off > 0; off >>= 1)
#pragma unroll
                for (int t = 0; t <= D; ++t) acc[t] = fe_add(acc[t], shfl_down_fe(acc[t], off));
        }
        if (q == 0 && threadIdx.x == 0) {
            fe rm;
            finalize_round<D, 0>(acc, round, ps, evals, chals, claim, &rm, nullptr, P.given);
            s_rm = rm;
        }
        cl.sync();                                    // r_i published; partials consumed
        const fe rm = *cl.map_shared_rank(&s_rm, 0);
#pragma unroll
        for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
        const uint32_t h = nl / 2;
        if (nl >= 4) {
            const uint32_t h2 = nl / 4;               // pairs of round i + 1
            for (uint32_t j = threadIdx.x; j < h2; j += blockDim.x) {
                fe a[D], bb[D];
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    const fe *T = cur + (size_t)m * nl;
                    fe *U = oth + (size_t)m * h;
                    if (ORDER == 0) {
                        a[m] = fold1(T[4 * j], T[4 * j + 1], rm);
                        bb[m] = fold1(T[4 * j + 2], T[4 * j + 3], rm);
                        U[2 * j] = a[m];
                        U[2 * j + 1] = bb[m];
                    } else {
                        a[m] = fold1(T[j], T[j + 2 * h2], rm);
                        bb[m] = fold1(T[j + h2], T[j + 3 * h2], rm);
                        U[j] = a[m];
                        U[j + h2] = bb[m];
                    }
                }
                eval_pair<D>(a, bb, acc);
            }
        } else if (threadIdx.x < D) {                 // nl == 2: the last local fold
            const fe *T = cur + (size_t)threadIdx.x * 2;
            oth[threadIdx.x] = fold1(T[0], T[1], rm);
        }
        __syncthreads();
        fe *tmp = cur; cur = oth; oth = tmp;
        nl = h;
    }
    // the last c rounds: the leader gathers entry q of every table from CTA q (global index q)
    cl.sync();
    if (q == 0 && threadIdx.x == 0) {
        fe one = fe_zero();
        one.l[0] = 1;
        for (uint32_t r = 0; r < CS; ++r) {
            const fe *rc = cl.map_shared_rank(cur, r);
#pragma unroll
            for (int m = 0; m < D; ++m) s_g[0][m][r] = rc[m];
        }
        int g = 0;
        for (uint32_t n = CS; n >= 2; n /= 2, ++round) {
            const uint32_t h = n / 2;
            fe acc[D + 1];
#pragma unroll
            for (int t = 0; t <= D; ++t) acc[t] = fe_zero();
            for (uint32_t j = 0; j < h; ++j) {
                fe a[D], bb[D];
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    a[m] = s_g[g][m][ORDER == 0 ? 2 * j : j];
                    bb[m] = s_g[g][m][ORDER == 0 ? 2 * j + 1 : j + h];
                }
                eval_pair<D>(a, bb, acc);
            }
            fe rm;
            finalize_round<D, 0>(acc, round, ps, evals, chals, claim, &rm, nullptr, P.given);
            for (uint32_t j = 0; j < h; ++j)
#pragma unroll
                for (int m = 0; m < D; ++m)
                    s_g[g ^ 1][m][j] = fold1(s_g[g][m][ORDER == 0 ? 2 * j : j], s_g[g][m][ORDER == 0 ? 2 * j + 1 : j + h], rm);
            g ^= 1;
        }
#pragma unroll
        for (int m = 0; m < D; ++m)
            st_fe(&P.final_evals[(size_t)b * D + m], m == 0 ? s_g[g][m][0] : mont_mul(s_g[g][m][0], one));
    }
    cl.sync();                                        // remote shared memory outlives the leader's reads
}

// k_impl.cuh (per degree)
template <int D>
cudaError_t launch_small(uint32_t order, dim3 grid, uint32_t cs, size_t smem, cudaStream_t s, const SmallParams &p);

}  // namespace bzk
