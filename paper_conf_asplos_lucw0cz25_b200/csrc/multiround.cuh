// multiround.cuh -- NEXT-1: the paper-literal sum-check (Alg. 1, d = 1) with KNOWN challenges,
// several rounds per pass over the table.
//
// PAPER.md:111 Alg. 1 takes r_1..r_n as inputs ("Random numbers r_1, ..., r_n"; produced by a
// PRG seeded with a Merkle root).  Without Fiat-Shamir nothing forces a barrier between rounds, so
// M rounds are done in ONE read of the table.  Take the current table A (2^K entries) and split the
// index into the M variables bound in the next M rounds (z, M bits) and the rest (y, K - M bits):
//   MSB (Alg. 1: round i pairs b, b + 2^{K-i}):  A[y + z 2^{K-M}],  round i binds bit z_{M-i}
//   LSB (north star: pairs 2j, 2j+1):             A[y 2^M + z],     round i binds bit z_{i-1}
// Folding is linear, so after the M rounds
//   A'[y] = sum_z w(z) A[y, z],        w(z) = prod_{i=1..M} (bit_i(z) ? r_i : 1 - r_i)
// (Alg. 1 line 5 applied M times), and the round sums of Alg. 1 lines 3-4 are, with the column sums
// C_z = sum_y A[y, z],
//   pi_i1 = sum_z [bit_i(z) = 0] w_{<i}(z) C_z,    pi_i2 = sum_z [bit_i(z) = 1] w_{<i}(z) C_z,
//   w_{<i}(z) = prod_{l<i} (bit_l(z) ? r_l : 1 - r_l).
// Per entry the kernel does one 256 x 256-bit product (weight w(z) R in Montgomery form, 544-bit
// unreduced accumulator, one reduction per output) and one 288-bit addition into C_z.  A pass reads
// the table once and writes 2^{-M} of it; each thread owns its column y, so MSB passes fold IN PLACE
// (A'[y] overwrites A[y + 0 * 2^{K-M}], read only by the same thread) -- Alg. 1's in-place update,
// race-free because of the ownership (P:165 needed two buffers for its streaming pipeline).
// Per-CTA partials of the 2^M column sums go through the last-CTA ticket as in k_round; the last CTA
// of a proof forms pi_i1, pi_i2 for the pass's M rounds (2^M M products) and writes them.
#pragma once
#include <stdint.h>
#include "field.cuh"
#include "sumcheck.cuh"

namespace bzk {

struct MultiParams {
    const fe *src;        // proof b's table: src + b * src_stride, 2^K entries (d = 1)
    fe *dst;              // proof b's output: dst + b * dst_stride, 2^(K-M) entries (MSB may fold in
                          // place: dst == src, dst_stride == src_stride)
    uint64_t src_stride, dst_stride;
    uint32_t logK;        // K: variables left before this pass
    uint32_t round0;      // first round of the pass (1-based)
    uint32_t k;           // total rounds
    uint32_t ctas;        // CTAs per proof
    fe *partials;         // [Bw][ctas][2^M]
    uint32_t *tickets;    // [Bw]
    const fe *challenges; // [Bw][k] (inputs)
    fe *round_evals;      // [Bw][k][2]
    fe *claims;           // [Bw] (may be null)
};

// The pass's round sums from the proof's column sums C_z (one thread): Alg. 1 lines 3-4 for the M
// rounds, pi_i1 / pi_i2 = sum over z with bit_i(z) = 0 / 1 of w_{<i}(z) C_z (header comment); the
// claim of round 1 is pi_11 + pi_12.  s_r holds r_i R and (1 - r_i) R.  (Inlined: as a separate call
// it produced wrong sums inside the kernels with dynamic shared memory -- B200 bring-up of k_multi_tc.)
template <int ORDER, int M>
__device__ __forceinline__ void multi_evals(const MultiParams &P, uint32_t b, const fe (&cs)[1 << M], const fe (&s_r)[M][2]) {
    constexpr int Z = 1 << M;
    fe *ev = P.round_evals + ((size_t)b * P.k + (P.round0 - 1)) * 2;
#pragma unroll 1
    for (int i = 1; i <= M; ++i) {
        fe g[2] = {fe_zero(), fe_zero()};
#pragma unroll 1
        for (int z = 0; z < Z; ++z) {
            fe c = fe_const(1);                           // w_{<i}(z) R
            for (int l = 1; l < i; ++l) {
                const int bit = ORDER == 1 ? (z >> (M - l)) & 1 : (z >> (l - 1)) & 1;
                c = mont_mul(c, s_r[l - 1][bit]);
            }
            const int bi = ORDER == 1 ? (z >> (M - i)) & 1 : (z >> (i - 1)) & 1;
            g[bi] = fe_add(g[bi], mont_mul(cs[z], c));
        }
        st_fe(ev + 2 * (i - 1), g[0]);
        st_fe(ev + 2 * (i - 1) + 1, g[1]);
        if (P.round0 == 1 && i == 1 && P.claims) st_fe(P.claims + b, fe_add(g[0], g[1]));
    }
}

// Pass setup shared by k_multi and k_multi_tc: s_r[i] = (r_i R, (1 - r_i) R) for the pass's rounds
// (threads < M), then s_w[z] = w(z) 2^288 mod p (threads < 2^M; acc17_to_fe_288 divides by 2^288).
template <int ORDER, int M>
__device__ __forceinline__ void multi_weights(const MultiParams &P, uint32_t b, fe (&s_r)[M][2], fe (&s_w)[1 << M]) {
    const fe *chal = P.challenges + (size_t)b * P.k + (P.round0 - 1);
    if (threadIdx.x < M) {
        const fe r = ld_fe(chal + threadIdx.x);
        s_r[threadIdx.x][1] = mont_mul(r, fe_const(2));                          // r R
        fe one = fe_zero();
        one.l[0] = 1;
        s_r[threadIdx.x][0] = mont_mul(fe_sub(one, r), fe_const(2));              // (1 - r) R
    }
    __syncthreads();
    if (threadIdx.x < (1u << M)) {
        fe w = fe_const(1);                                                       // R = 1 in Montgomery form
#pragma unroll
        for (int i = 1; i <= M; ++i) {
            const int bit = ORDER == 1 ? (threadIdx.x >> (M - i)) & 1 : (threadIdx.x >> (i - 1)) & 1;
            w = mont_mul(w, s_r[i - 1][bit]);
        }
        fe c288 = fe_const(1);                                                    // 2^256 mod p
        for (int e = 0; e < 32; ++e) c288 = fe_add(c288, c288);                 // 2^288 mod p
        s_w[threadIdx.x] = mont_mul(w, c288);                                     // (w R) 2^288 / R = w 2^288
    }
    __syncthreads();
}

// TMA = true (MSB only): the warp's 32 columns are streamed into shared memory segment by segment --
// segment z holds entry z of the 32 columns, the 1 KiB A[y0 + z 2^(K-M) .. + 31] -- and each segment's
// copy for the next grid-stride block is issued as soon as every lane has consumed it (sumcheck.cuh
// TMA helpers; 128-byte swizzle, conflict-free LDS), so one entry at a time is live in registers.
template <int ORDER, int M, bool TMA>
__global__ void __launch_bounds__(256, 2) k_multi(MultiParams P, const __grid_constant__ CUtensorMap tmap) {
    constexpr int Z = 1 << M;
    __shared__ fe s_w[Z];              // w(z) 2^288 (acc17_to_fe_288 divides the row sums by 2^288)
    __shared__ fe s_r[M][2];           // r_i R, (1 - r_i) R
    __shared__ fe s_red[32 * Z];
    __shared__ int s_last;
    const uint32_t b = blockIdx.y;
    multi_weights<ORDER, M>(P, b, s_r, s_w);

    const uint64_t Ny = 1ull << (P.logK - M);         // outputs (columns) per proof
    const fe *src = P.src + (size_t)b * P.src_stride;
    fe *dst = P.dst + (size_t)b * P.dst_stride;
    const uint64_t stride = (uint64_t)P.ctas * blockDim.x;
    fe col[Z];                                         // column sums, lazy: < 2p
#pragma unroll
    for (int z = 0; z < Z; ++z) col[z] = fe_zero();
    if constexpr (TMA) {
        static_assert(ORDER == 1, "TMA staging of k_multi is built for the MSB (Alg. 1) layout");
        extern __shared__ uint8_t tma_raw[];
        __shared__ __align__(8) uint64_t bars[8 * Z];
        uint8_t *tma_base = tma_raw + ((1024 - (smem_u32(tma_raw) & 1023)) & 1023);
        const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
        uint8_t *seg = tma_base + (size_t)warp * Z * 1024;
        uint64_t *wb = bars + warp * Z;
        if (lane == 0) {
#pragma unroll
            for (int z = 0; z < Z; ++z) mbar_init(&wb[z]);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncwarp();
        const uint64_t row0 = (uint64_t)b * P.src_stride / 4;     // 4 entries of 32 B per 128-byte row
        const uint64_t y0 = (uint64_t)blockIdx.x * blockDim.x + warp * 32;
        auto issue = [&](int z, uint64_t yb) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&wb[z], 1024);
            tma_load_rows(seg + z * 1024, &tmap, row0 + (yb + (uint64_t)z * Ny) / 4, &wb[z]);
        };
        if (lane == 0 && y0 < Ny)
#pragma unroll
            for (int z = 0; z < Z; ++z) issue(z, y0);
        uint32_t it = 0;
        for (uint64_t yw = y0; yw < Ny; yw += stride, ++it) {
            acc17 acc = acc17_zero();
#pragma unroll
            for (int z = 0; z < Z; ++z) {
                mbar_wait(&wb[z], it & 1);
                const uint32_t row = lane >> 2, c0 = 2 * (lane & 3);
                const uint8_t *base = seg + z * 1024 + row * 128;
                const uint4 lo = *reinterpret_cast<const uint4 *>(base + ((c0 ^ (row & 7)) << 4));
                const uint4 hi = *reinterpret_cast<const uint4 *>(base + (((c0 + 1) ^ (row & 7)) << 4));
                fe x;
                x.l[0] = lo.x; x.l[1] = lo.y; x.l[2] = lo.z; x.l[3] = lo.w;
                x.l[4] = hi.x; x.l[5] = hi.y; x.l[6] = hi.z; x.l[7] = hi.w;
                col[z] = lz_red(lz_add(col[z], x));
                mul_acc(acc, s_w[z], x);
                __syncwarp();                          // every lane has used segment z
                if (lane == 0 && yw + stride < Ny) issue(z, yw + stride);
            }
            st_fe(dst + yw + lane, acc17_to_fe_288(acc));
        }
    } else
    for (uint64_t y = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; y < Ny; y += stride) {
        fe x[Z];
#pragma unroll
        for (int z = 0; z < Z; ++z) x[z] = ld_fe_stream(src + (ORDER == 1 ? y + (uint64_t)z * Ny : (y << M) + z));
        acc17 acc = acc17_zero();
#pragma unroll
        for (int z = 0; z < Z; ++z) {
            col[z] = lz_red(lz_add(col[z], x[z]));    // < 2p + p, minus 2p when >= 2p
            mul_acc(acc, s_w[z], x[z]);
        }
        st_fe(dst + y, acc17_to_fe_288(acc));          // canonical: A'[y] = sum_z w(z) A[y, z]
    }

    // column sums of the proof: thread -> block -> per-CTA partial -> last-CTA ticket
    fe cs[Z];
#pragma unroll
    for (int z = 0; z < Z; ++z) cs[z] = fe_reduce_once(col[z]);
    block_reduce<Z>(cs, s_red);
    fe *part = P.partials + (size_t)b * P.ctas * Z;
    if (P.ctas > 1) {
        if (threadIdx.x == 0) {
#pragma unroll
            for (int z = 0; z < Z; ++z) st_fe_cg(&part[(size_t)blockIdx.x * Z + z], cs[z]);
            __threadfence();
            s_last = atomicAdd(&P.tickets[b], 1u) == P.ctas - 1;
        }
        __syncthreads();
        if (!s_last) return;
        __threadfence();
#pragma unroll
        for (int z = 0; z < Z; ++z) cs[z] = fe_zero();
        for (uint32_t c = threadIdx.x; c < P.ctas; c += blockDim.x)
#pragma unroll
            for (int z = 0; z < Z; ++z) cs[z] = fe_add(cs[z], ld_fe_cg(&part[(size_t)c * Z + z]));
        block_reduce<Z>(cs, s_red);
    }
    if (threadIdx.x != 0) return;
    if (P.ctas > 1) P.tickets[b] = 0;
    multi_evals<ORDER, M>(P, b, cs, s_r);
}

// k_multi.cu
cudaError_t multi_launch(uint32_t order, uint32_t m, bool tma, dim3 grid, cudaStream_t s, const MultiParams &p,
                         const CUtensorMap &tm);
cudaError_t multi_set_attrs();
// k_multi_tc (multiround_tc.cuh): three rounds per pass, 128-column tiles, tensor-core row sums
constexpr uint32_t kTcTileRows = 128;   // columns y per tile (the MMA's M)
cudaError_t multi_tc_launch(uint32_t order, dim3 grid, cudaStream_t s, const MultiParams &p, const CUtensorMap &tm);

}  // namespace bzk
