// multiround_tc.cuh -- the known-challenge pass of three rounds (NEXT-1, multiround.cuh) with the
// weighted row sums on the tensor cores (tcgen05 kind::i8).
//
// The pass computes, for every column y of a proof's table A (2^K entries, Ny = 2^(K-3) columns),
//   A'[y] = sum_z w(z) A[y, z]     (z = the 3 bound variables; multiround.cuh header, reading R26)
// and the column sums C_z = sum_y A[y, z] that give Alg. 1's round sums.
// Both are integer contractions over bytes.  With x_z = A[y, z] = sum_i a_{z,i} 2^(8i) (32 bytes) and
// W_z = w(z) 2^288 mod p = sum_j b_{z,j} 2^(8j), the 511-bit integer
//   S(y) = sum_z W_z x_z = sum_n c_n 2^(8n),   c_n = sum_z sum_{i+j=n} a_{z,i} b_{z,j}  (< 2^24)
// is one u8 x u8 -> s32 matrix product per 128-column tile: D[y][n] = sum_(z,i) a[y][(z,i)] B[n][(z,i)]
// with the Toeplitz operand B[n][(z,i)] = b_{z,n-i} (0 outside 0..31), M = 128, N = 64, K = 8 x 32.
// The epilogue carries the 63 column values into 16 words and reduces once (acc17_to_fe_288, the
// same 9-word REDC k_multi uses), so every output is the canonical A'[y] bit for bit.  The column
// byte sums are a second product with an all-ones operand, D2[.][(z,i)] = sum_y a[y][(z,i)]
// (the tile read MN-major, N = 256, K = y), accumulated in TMEM over all the CTA's tiles; C_z =
// sum_i D2[(z,i)] 2^(8i).  So the integer pipe does ~30 operations per entry instead of a 256 x 256-bit
// product, and the pass streams at the HBM rate.
//
// Roles (one CTA per SM, 64 + 128 EG threads): warp 0 issues the TMA loads (one 32 KiB stage = the 8
// segments of 128 entries, 32-byte rows, 32-byte swizzle), warp 1 owns TMEM and issues the MMAs,
// warps 2.. are EG epilogue groups of four warps (group g takes the tiles it = g mod EG and TMEM
// accumulator g; warp w reads TMEM lanes 32 (w mod 4) ..).  MSB folds in place as k_multi does: the
// output row y overwrites A[y + 0 Ny], which only this CTA's tile y reads, and only before.
#pragma once
#include <stdint.h>
#include "multiround.cuh"
#include "tc.cuh"

namespace bzk {

// NS: 32 KiB TMA stages; EG: epilogue groups of 4 warps (one 64-column TMEM accumulator each, <= 4);
// CM: M of the column-sum product (64 or 128 rows of ones: every row of D2 is the same vector, row 0
// sits in TMEM lane 0 either way)
constexpr int tc_threads(int EG) { return 64 + 128 * EG; }
constexpr size_t tc_smem(int NS) { return 1024 + (size_t)NS * 32768 + 16384 + 4096; }   // + B operand + ones

template <int ORDER, int NS, int EG, int CM>
__global__ void __launch_bounds__(tc_threads(EG), 1) k_multi_tc(MultiParams P, const __grid_constant__ CUtensorMap tmap) {
    static_assert(EG >= 1 && EG <= 4 && (CM == 64 || CM == 128), "k_multi_tc shape");
    constexpr int M = 3, Z = 8, kTcStages = NS;
    __shared__ fe s_w[Z];
    __shared__ fe s_r[M][2];
    __shared__ fe s_cs[Z];
    __shared__ __align__(8) uint64_t full[kTcStages], empty[kTcStages], tfull[EG], tempty[EG], dfin;
    __shared__ uint32_t s_tmem;
    __shared__ int s_last;
    extern __shared__ uint8_t tc_raw[];
    uint8_t *base = tc_raw + ((1024 - (tc::su32(tc_raw) & 1023)) & 1023);
    uint8_t *stage0 = base;                                    // [stage][z][128 rows][32 B], swizzled
    uint8_t *opB = base + kTcStages * 32768;                   // [z][64 rows n][32 B], swizzled
    uint8_t *ones = opB + 16384;                               // 128 x 32 bytes of 1
    BZK_ASSERT((size_t)(ones + 4096 - tc_raw) <= dyn_smem_bytes());
    const uint32_t b = blockIdx.y, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    multi_weights<ORDER, M>(P, b, s_r, s_w);
    // Toeplitz B operand: row n, chunk h of segment z holds bytes b_{z, n - i}, i = 16 h .. 16 h + 15
    for (uint32_t c = threadIdx.x; c < Z * 64 * 2; c += blockDim.x) {
        const uint32_t z = c >> 7, n = (c >> 1) & 63, h = c & 1;
        uint32_t q[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
            uint32_t v = 0;
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                const int j = (int)n - (int)(h * 16 + e * 4 + t);
                const uint32_t by = (j >= 0 && j < 32) ? (s_w[z].l[j >> 2] >> (8 * (j & 3))) & 255u : 0u;
                v |= by << (8 * t);
            }
            q[e] = v;
        }
        *reinterpret_cast<uint4 *>(opB + z * 2048 + n * 32 + ((h ^ ((n >> 2) & 1)) << 4)) = make_uint4(q[0], q[1], q[2], q[3]);
    }
    for (uint32_t c = threadIdx.x; c < 4096 / 16; c += blockDim.x)
        *reinterpret_cast<uint4 *>(ones + c * 16) = make_uint4(0x01010101u, 0x01010101u, 0x01010101u, 0x01010101u);
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTcStages; ++s) { tc::mbar_init_n(&full[s], 1); tc::mbar_init_n(&empty[s], 1); }
        for (int g = 0; g < EG; ++g) { tc::mbar_init_n(&tfull[g], 1); tc::mbar_init_n(&tempty[g], 128); }
        tc::mbar_init_n(&dfin, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) tc::tmem_alloc<512>(&s_tmem);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // B / ones (generic writes) -> MMA reads
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;

    const uint32_t Ny = 1u << (P.logK - M);
    const uint32_t T = Ny / kTcTileRows;                       // tiles of this proof
    const uint32_t nt = blockIdx.x < T ? (T - 1 - blockIdx.x) / P.ctas + 1 : 0;   // this CTA's tiles

    if (warp == 0) {
        if (lane == 0) {
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % kTcStages;
                if (it >= (uint32_t)kTcStages) tc::mbar_wait(&empty[s], ((it / kTcStages) - 1) & 1);
                const int y0 = (int)((blockIdx.x + it * P.ctas) * kTcTileRows);
                uint8_t *st = stage0 + s * 32768;
                tc::mbar_tx(&full[s], 32768);
                if (ORDER == 1) {
                    tc::tma4(st, &tmap, 0, y0, 0, (int)b, &full[s]);        // dims (8 w, Ny, Z, B): [z][y] in one box
                } else {
#pragma unroll
                    for (int z = 0; z < Z; ++z) tc::tma4(st + z * 4096, &tmap, 0, z, y0, (int)b, &full[s]);   // (8 w, Z, Ny, B)
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            const uint32_t id_main = tc::idesc_u8(128, 64, false), id_col = tc::idesc_u8(CM, 256, true);
            const uint32_t sb = tc::su32(stage0), bb = tc::su32(opB), ob = tc::su32(ones);
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % kTcStages, g = it % EG;
                tc::mbar_wait(&full[s], (it / kTcStages) & 1);
                if (it >= (uint32_t)EG) tc::mbar_wait(&tempty[g], ((it / EG) - 1) & 1);
                tc::fence_after();
                const uint32_t a0 = sb + s * 32768;
#pragma unroll
                for (int z = 0; z < Z; ++z)
                    tc::mma_u8(tmem + g * 64, tc::desc_sw32(a0 + z * 4096, 16, 256), tc::desc_sw32(bb + z * 2048, 16, 256),
                               id_main, z > 0);
#pragma unroll
                for (int q = 0; q < 4; ++q)   // column byte sums: K = 32 rows y per instruction
                    tc::mma_u8(tmem + 256, tc::desc_sw32(ob, 16, 256), tc::desc_sw32(a0 + q * 1024, 4096, 256), id_col,
                               it > 0 || q > 0);
                tc::commit(&empty[s]);
                tc::commit(&tfull[g]);
            }
            if (nt > 0) tc::commit(&dfin);
        }
        __syncwarp();
    } else {
        const uint32_t e = warp - 2, g = e >> 2, qd = warp & 3, row = qd * 32 + lane;
        const uint32_t ta = tmem + ((qd * 32) << 16) + g * 64;
        fe *dst = P.dst + (size_t)b * P.dst_stride;
        for (uint32_t it = g; it < nt; it += EG) {
            tc::mbar_wait(&tfull[g], (it / EG) & 1);
            tc::fence_after();
            uint32_t c0[32], c1[32];
            tc::ld_x32(ta, c0);
            tc::ld_x32(ta + 32, c1);
            tc::wait_ld();
            tc::fence_before();
            tc::mbar_arrive(&tempty[g]);
            // S = sum_n c_n 2^(8n) -> 16 words (S < 8 p 2^256 < 2^511)
            acc17 S;
            uint64_t carry = 0;
#pragma unroll
            for (int j = 0; j < 16; ++j) {
                const uint32_t *c = j < 8 ? c0 + 4 * j : c1 + 4 * (j - 8);
                const uint64_t v = carry + c[0] + ((uint64_t)c[1] << 8) + ((uint64_t)c[2] << 16) + ((uint64_t)c[3] << 24);
                S.w[j] = (uint32_t)v;
                carry = v >> 32;
            }
            S.w[16] = (uint32_t)carry;
            const uint32_t y = (blockIdx.x + it * P.ctas) * kTcTileRows + row;
            st_fe(dst + y, acc17_to_fe_288(S));                 // canonical A'[y] = sum_z w(z) A[y, z]
        }
        if (warp == 4) {                                        // group 0, TMEM lanes 0..31: the column sums
            fe cz = fe_zero();
            if (nt > 0) {
                tc::mbar_wait(&dfin, 0);
                tc::fence_after();
#pragma unroll 1
                for (int z = 0; z < Z; ++z) {
                    uint32_t v[32];
                    tc::ld_x32(tmem + 256 + z * 32, v);        // every row of D2 is the same byte-sum vector
                    tc::wait_ld();
                    if (lane == (uint32_t)z) {
                        acc9 a;
                        uint64_t carry = 0;
#pragma unroll
                        for (int j = 0; j < 8; ++j) {
                            const uint64_t s = carry + v[4 * j] + ((uint64_t)v[4 * j + 1] << 8) +
                                               ((uint64_t)v[4 * j + 2] << 16) + ((uint64_t)v[4 * j + 3] << 24);
                            a.lo.l[j] = (uint32_t)s;
                            carry = s >> 32;
                        }
                        a.hi = (uint32_t)carry;
                        cz = acc9_to_fe(a);                     // C_z mod p (Montgomery form of the sum)
                    }
                }
            }
            tc::fence_before();
            if (lane < (uint32_t)Z) s_cs[lane] = cz;
        }
    }
    __syncthreads();
    if (warp == 1) {
        tc::fence_after();
        tc::tmem_dealloc<512>(tmem);
    }
    if (warp != 4) return;
    // per-CTA column sums -> last-CTA ticket -> the pass's round sums (as k_multi)
    fe *part = P.partials + (size_t)b * P.ctas * Z;
    fe cs[Z];
    if (P.ctas > 1) {
        if (lane < (uint32_t)Z) st_fe_cg(&part[(size_t)blockIdx.x * Z + lane], s_cs[lane]);
        __threadfence();
        __syncwarp();
        if (lane == 0) s_last = atomicAdd(&P.tickets[b], 1u) == P.ctas - 1;
        __syncwarp();
        if (!s_last) return;
        __threadfence();
        if (lane < (uint32_t)Z) {
            fe a = fe_zero();
            for (uint32_t c = 0; c < P.ctas; ++c) a = fe_add(a, ld_fe_cg(&part[(size_t)c * Z + lane]));
            s_cs[lane] = a;
        }
        __syncwarp();
    }
    if (lane != 0) return;
    if (P.ctas > 1) P.tickets[b] = 0;
#pragma unroll
    for (int z = 0; z < Z; ++z) cs[z] = s_cs[z];
    multi_evals<ORDER, M>(P, b, cs, s_r);
}

}  // namespace bzk
