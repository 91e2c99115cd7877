// round1_tc.cuh -- round 1 of the degree-2 sum-check on the tensor cores (tcgen05 kind::i8).
//
// Round 1 (Alg. 1 lines 3-4 generalised to a product of d = 2 multilinears, SURVEY.md
// 8(a2)) sums, over the h = 2^(k-1) pairs j of a proof, the products of the two tables' values at the
// summed points (sumcheck.cuh Pts<2, FIRST>): g(0) = sum_j a0_j a1_j, g(1) = sum_j b0_j b1_j and the
// leading coefficient c_inf = sum_j (b0_j - a0_j)(b1_j - a1_j) (a = entry 2j / j, b = 2j+1 / j+h for
// LSB / MSB).  Every such sum is a bilinear form over bytes: with x_j = sum_i x_{j,i} 2^(8i),
//   sum_j x_j y_j = sum_{i,i'} M[i][i'] 2^(8(i+i')),    M = X^T Y,  X, Y = [pairs j] x [32 bytes],
// a u8 matrix product whose contraction runs over the pairs (K = j).  One MMA per 32 pairs computes
// the four block sums S_aa, S_ab, S_ba, S_bb of (a0 | b0) x (a1 | b1) straight from the TMA tiles:
// A = the bytes of (a1 | b1 | a0 | b0) as 128 rows (MN-major: each pair's 32 bytes are contiguous),
// B = (a1 | b1) -- the same first 64 rows -- as 64 columns; D rows 64..127 are the blocks (rows 0..63,
// a1 | b1 against itself, are not used).  Then g(0) = S_aa, g(1) = S_bb and
// c_inf = S_bb - S_ab - S_ba + S_aa (mod p): the same residues as summing (b0 - a0)(b1 - a1), with no
// per-pair subtraction on the SMs.
//
// s32 accumulators: 16384 pairs per TMEM accumulation chunk keep every M entry < 16384 * 255^2 < 2^31;
// the epilogue warps add each finished chunk (two TMEM buffers) into 64-bit registers.  After the
// CTA's last tile: the anti-diagonal sums s_n = sum_{i+i'=n} M[i][i'] (< 2^43), S = sum_n s_n 2^(8n)
// (< 2^544, 17 words), acc17_to_fe(S) = S R^-1 mod p per block -- the per-CTA partials k_round's acc17
// path produces up to the block combination -- then round_finish (ticket, transcript, r_1, outputs) as
// every global round.
//
// Roles (1 CTA per SM, 128 threads): warp 0 TMA (a and b tiles of both tables, 32-byte rows, 32-byte
// swizzle), warp 1 TMEM + MMA issue, warps 2 / 3 the epilogue (TMEM lanes 64..95 / 96..127: the a0 /
// b0 rows, 64 columns each).
#pragma once
#include <stdint.h>
#include "sumcheck.cuh"
#include "tc.cuh"

namespace bzk {

// NS: 16 KiB stages ([a1][b1][a0][b0] x 128 pairs)
constexpr uint32_t kR1Tile = 128;                  // pairs per tile
constexpr uint32_t kR1Chunk = 128;                 // tiles per TMEM accumulation chunk (16384 pairs)
constexpr uint32_t kR1Stage = 16384;
constexpr int kR1Threads = 128;
constexpr size_t r1_smem(int NS) { return 1024 + (size_t)NS * kR1Stage; }

// SW64 (LSB only): the stage holds each table's 128 pairs as contiguous 64-byte rows (a_j | b_j), one TMA
// box of 8 KiB per table with the 64-byte swizzle, read by the MMA as 64-element MN blocks (the byte
// rows 0..63 / 64..127 of A and the columns of B are the same (a | b) vectors as in the 32-byte
// layout); otherwise a and b arrive as separate 4 KiB boxes of 32-byte rows (LSB: every other entry).
template <int ORDER, int NS, bool SW64>
__global__ void __launch_bounds__(kR1Threads, 1) k_round1_tc(RoundParams P, const __grid_constant__ CUtensorMap tmap) {
    static_assert(!SW64 || ORDER == 0, "64-byte rows (a_j | b_j) exist in LSB order only");
    constexpr int D = 2, NV = Pts<2, false>::NV;   // points 0, 1, inf
    __shared__ fe s_red[32 * NV];
    __shared__ fe s_clu[NV];
    __shared__ int s_last;
    __shared__ __align__(8) uint64_t full[NS], empty[NS], dready[2], dempty[2];
    __shared__ uint32_t s_tmem;
    __shared__ unsigned long long s_diag[4][64];   // blocks aa, ab, ba, bb
    extern __shared__ uint8_t r1_raw[];
    uint8_t *base = r1_raw + ((1024 - (tc::su32(r1_raw) & 1023)) & 1023);
    BZK_ASSERT((size_t)(base - r1_raw) + (size_t)NS * kR1Stage <= dyn_smem_bytes());
    const uint32_t b = blockIdx.y, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t h = 1ull << P.log_h;
    const uint32_t T = (uint32_t)(h / kR1Tile);
    const uint32_t nt = blockIdx.x < T ? (T - 1 - blockIdx.x) / P.ctas + 1 : 0;
    const uint32_t nch = (nt + kR1Chunk - 1) / kR1Chunk;

    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) {
            tc::mbar_init_n(&full[s], 1);
            tc::mbar_init_n(&empty[s], 1);
        }
        for (int g = 0; g < 2; ++g) { tc::mbar_init_n(&dready[g], 1); tc::mbar_init_n(&dempty[g], 64); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) tc::tmem_alloc<128>(&s_tmem);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    unsigned long long macc[64];                   // epilogue: this row's 64 M entries (64-bit)
#pragma unroll
    for (int i = 0; i < 64; ++i) macc[i] = 0;

    if (warp == 0) {
        if (lane == 0) {
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % NS;
                if (it >= (uint32_t)NS) tc::mbar_wait(&empty[s], ((it / NS) - 1) & 1);
                const int j0 = (int)((blockIdx.x + it * P.ctas) * kR1Tile);
                BZK_ASSERT((uint64_t)j0 + kR1Tile <= h);
                uint8_t *st = base + s * kR1Stage;
                tc::mbar_tx(&full[s], kR1Stage);
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    const int tab = (int)(b * D + m);
                    uint8_t *dstm = st + (1 - m) * 8192;   // table 1 first: A = (a1 | b1 | a0 | b0)
                    if (SW64) {         // dims (16 w, h, tables): rows (a_j | b_j)
                        tc::tma3(dstm, &tmap, 0, j0, tab, &full[s]);
                    } else if (ORDER == 1) {   // dims (8 w, h, 2: a / b, tables): a and b tiles in one box
                        tc::tma4(dstm, &tmap, 0, j0, 0, tab, &full[s]);
                    } else {            // dims (8 w, 2: a / b, h, tables)
                        tc::tma4(dstm, &tmap, 0, 0, j0, tab, &full[s]);
                        tc::tma4(dstm + 4096, &tmap, 0, 1, j0, tab, &full[s]);
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            const uint32_t idesc = tc::idesc_u8(128, 64, true) | (1u << 15);   // A and B MN-major
            const uint32_t sb = tc::su32(base);
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % NS, c = it / kR1Chunk, g = c & 1, first = it % kR1Chunk == 0;
                tc::mbar_wait(&full[s], (it / NS) & 1);
                if (first && c >= 2) tc::mbar_wait(&dempty[g], ((c >> 1) - 1) & 1);
                tc::fence_after();
                const uint32_t a0 = sb + s * kR1Stage;
#pragma unroll
                for (int q = 0; q < 4; ++q) {   // K = 32 pairs per instruction
                    const uint64_t da = SW64 ? tc::desc_sw64(a0 + q * 2048, 8192, 512) : tc::desc_sw32(a0 + q * 1024, 4096, 256);
                    tc::mma_u8(tmem + g * 64, da, da, idesc, !(first && q == 0));
                }
                tc::commit(&empty[s]);
                if (it % kR1Chunk == kR1Chunk - 1 || it == nt - 1) tc::commit(&dready[g]);
            }
        }
        __syncwarp();
    } else {
        // warp 2: TMEM lanes 64..95 (byte i of a0), warp 3: lanes 96..127 (byte i of b0); columns 0..31
        // pair them with a1, 32..63 with b1
        for (uint32_t c = 0; c < nch; ++c) {
            const uint32_t g = c & 1;
            tc::mbar_wait(&dready[g], (c >> 1) & 1);
            tc::fence_after();
#pragma unroll
            for (int half = 0; half < 2; ++half) {
                uint32_t v[32];
                tc::ld_x32(tmem + ((warp * 32) << 16) + g * 64 + half * 32, v);
                tc::wait_ld();
#pragma unroll
                for (int i = 0; i < 32; ++i) macc[half * 32 + i] += v[i];
            }
            tc::fence_before();
            tc::mbar_arrive(&dempty[g]);
        }
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 1) {
        tc::fence_after();
        tc::tmem_dealloc<128>(tmem);
    }
    // anti-diagonal sums s_n = sum_{i+i'=n} M[i][i'] of the four blocks, then S -> acc17 -> fe
    for (uint32_t q = threadIdx.x; q < 4 * 64; q += blockDim.x) s_diag[q >> 6][q & 63] = 0;
    __syncthreads();
    if (warp >= 2) {
        const uint32_t r = warp - 2;               // 0: a0 rows, 1: b0 rows
#pragma unroll
        for (int half = 0; half < 2; ++half)       // 0: x a1, 1: x b1
#pragma unroll
            for (int i = 0; i < 32; ++i)
                atomicAdd(&s_diag[2 * r + half][lane + i], macc[half * 32 + i]);
    }
    __syncthreads();
    __shared__ fe s_blk[4];
    if (threadIdx.x < 4) {
        fe f = fe_zero();
        if (nt > 0) {
            acc17 S = acc17_zero();
            for (int n = 0; n < 63; ++n) {   // add s_n 2^(8n): 64-bit value at bit offset 8n
                const unsigned long long v = s_diag[threadIdx.x][n];
                const int w0 = (8 * n) >> 5, sh = (8 * n) & 31;
                uint64_t cur = (uint64_t)S.w[w0] + (uint32_t)(v << sh);
                S.w[w0] = (uint32_t)cur;
                uint64_t carry = (cur >> 32) + (sh ? (v >> (32 - sh)) : (v >> 32));   // < 2^44
                for (int w = w0 + 1; w < 17 && carry; ++w) {
                    cur = (uint64_t)S.w[w] + (uint32_t)carry;
                    S.w[w] = (uint32_t)cur;
                    carry = (carry >> 32) + (cur >> 32);
                }
            }
            f = acc17_to_fe(S);
        }
        s_blk[threadIdx.x] = f;                    // aa, ab, ba, bb (each S R^-1 mod p, canonical)
    }
    __syncthreads();
    // Pts<2, FIRST> order: 0 -> g(0) = aa, 1 -> g(1) = bb, 2 -> c_inf = bb - ab - ba + aa
    fe acc[NV];
    acc[0] = s_blk[0];
    acc[1] = s_blk[3];
    acc[2] = fe_add(fe_sub(fe_sub(s_blk[3], s_blk[1]), s_blk[2]), s_blk[0]);
    if (threadIdx.x != 0) {
#pragma unroll
        for (int t = 0; t < NV; ++t) acc[t] = fe_zero();
    }
    round_finish<D, false>(P, b, acc, s_red, s_clu, &s_last);
}

}  // namespace bzk
