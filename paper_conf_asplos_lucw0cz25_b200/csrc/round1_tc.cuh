// round1_tc.cuh -- round 1 of the degree-2 sum-check on the tensor cores (tcgen05 kind::i8).
//
// Round 1 (Alg. 1 lines 3-4 generalised to a product of d = 2 multilinears, SURVEY.md
// 8(a2)) sums, over the h = 2^(k-1) pairs j of a proof, the products of the two tables' values at the
// summed points (sumcheck.cuh Pts<2, FIRST>): g(0) = sum_j a0_j a1_j, g(1) = sum_j b0_j b1_j and the
// leading coefficient c_inf = sum_j D0_j D1_j with D = b - a (a = entry 2j / j, b = 2j+1 / j+h for
// LSB / MSB).  Every such sum is a bilinear form over bytes: with x_j = sum_i x_{j,i} 2^(8i),
//   sum_j x_j y_j = sum_{i,i'} M[i][i'] 2^(8(i+i')),    M = X^T Y,  X, Y = [pairs j] x [32 bytes],
// a u8 matrix product whose contraction runs over the pairs (K = j).  One MMA per 32 pairs computes
// all three: A = the bytes of (a0 | b0 | D0 | -) as 128 rows (MN-major: each pair's 32 bytes are
// contiguous), B = the bytes of (a1 | b1 | D1) as 96 columns; the diagonal 32 x 32 blocks of
// D[128][96] are the three M's (the off-diagonal blocks and rows 96..127 are not used).  D = b + p - a
// in [1, 2p) keeps the operand non-negative and < 2^256 (the product's residue is that of (b - a)^2
// terms, so the sums match k_round's exactly mod p).
//
// s32 accumulators: 16384 pairs per TMEM accumulation chunk keep every M entry < 16384 * 255^2 < 2^31;
// the epilogue warps add each finished chunk (two TMEM buffers) into 64-bit registers.  After the
// CTA's last tile: the anti-diagonal sums s_n = sum_{i+i'=n} M[i][i'] (< 2^43), S = sum_n s_n 2^(8n)
// (< 2^544, 17 words), acc17_to_fe(S) = S R^-1 mod p -- the same canonical per-CTA partial k_round's
// acc17 path produces -- then round_finish (ticket, transcript, r_1, outputs) as every global round.
//
// Roles (1 CTA per SM, 32 (6 + PW) threads): warp 0 TMA (a and b tiles of both tables, 32-byte rows,
// 32-byte swizzle), warp 1 TMEM + MMA issue, PW warps form D = b + p - a in shared memory, the last 4 warps
// the epilogue (warp w reads TMEM lanes 32 (w mod 4): rows 0..95 = the a, b, D blocks).
#pragma once
#include <stdint.h>
#include "sumcheck.cuh"
#include "tc.cuh"

namespace bzk {

// NS: 24 KiB stages ([a0][b0][D0][a1][b1][D1] x 128 pairs); PW: D-prep warps (2 or 4)
constexpr uint32_t kR1Tile = 128;                  // pairs per tile
constexpr uint32_t kR1Chunk = 128;                 // tiles per TMEM accumulation chunk (16384 pairs)
constexpr int r1_threads(int PW) { return 32 * (2 + PW + 4); }
constexpr size_t r1_smem(int NS) { return 1024 + (size_t)NS * 24576; }

template <int ORDER, int NS, int PW>
__global__ void __launch_bounds__(r1_threads(PW), 1) k_round1_tc(RoundParams P, const __grid_constant__ CUtensorMap tmap) {
    constexpr int D = 2, NV = Pts<2, false>::NV;   // points 0, 1, inf
    constexpr int kR1Stages = NS;
    static_assert(PW == 2 || PW == 4, "D-prep warps");
    __shared__ fe s_red[32 * NV];
    __shared__ fe s_clu[NV];
    __shared__ int s_last;
    __shared__ __align__(8) uint64_t full[kR1Stages], prep[kR1Stages], empty[kR1Stages], dready[2], dempty[2];
    __shared__ uint32_t s_tmem;
    __shared__ unsigned long long s_diag[3][64];
    extern __shared__ uint8_t r1_raw[];
    uint8_t *base = r1_raw + ((1024 - (tc::su32(r1_raw) & 1023)) & 1023);
    const uint32_t b = blockIdx.y, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t h = 1ull << P.log_h;
    const uint32_t T = (uint32_t)(h / kR1Tile);
    const uint32_t nt = blockIdx.x < T ? (T - 1 - blockIdx.x) / P.ctas + 1 : 0;
    const uint32_t nch = (nt + kR1Chunk - 1) / kR1Chunk;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kR1Stages; ++s) {
            tc::mbar_init_n(&full[s], 1);
            tc::mbar_init_n(&prep[s], 32 * PW);
            tc::mbar_init_n(&empty[s], 1);
        }
        for (int g = 0; g < 2; ++g) { tc::mbar_init_n(&dready[g], 1); tc::mbar_init_n(&dempty[g], 128); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) tc::tmem_alloc<256>(&s_tmem);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    unsigned long long macc[32];                   // epilogue: this row's 32 M entries (64-bit)
#pragma unroll
    for (int i = 0; i < 32; ++i) macc[i] = 0;

    if (warp == 0) {
        if (lane == 0) {
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % kR1Stages;
                if (it >= (uint32_t)kR1Stages) tc::mbar_wait(&empty[s], ((it / kR1Stages) - 1) & 1);
                const int j0 = (int)((blockIdx.x + it * P.ctas) * kR1Tile);
                uint8_t *st = base + s * 24576;
                tc::mbar_tx(&full[s], 4 * 4096);
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    const int tab = (int)(b * D + m);
                    if (ORDER == 1) {   // dims (8 w, h, 2: a / b, tables): a and b tiles in one box
                        tc::tma4(st + m * 12288, &tmap, 0, j0, 0, tab, &full[s]);
                    } else {            // dims (8 w, 2: a / b, h, tables)
                        tc::tma4(st + m * 12288, &tmap, 0, 0, j0, tab, &full[s]);
                        tc::tma4(st + m * 12288 + 4096, &tmap, 0, 1, j0, tab, &full[s]);
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            const uint32_t idesc = tc::idesc_u8(128, 96, true) | (1u << 15);   // A and B MN-major
            const uint32_t sb = tc::su32(base);
            for (uint32_t it = 0; it < nt; ++it) {
                const uint32_t s = it % kR1Stages, c = it / kR1Chunk, g = c & 1, first = it % kR1Chunk == 0;
                tc::mbar_wait(&prep[s], (it / kR1Stages) & 1);
                if (first && c >= 2) tc::mbar_wait(&dempty[g], ((c >> 1) - 1) & 1);
                tc::fence_after();
                const uint32_t a0 = sb + s * 24576;
#pragma unroll
                for (int q = 0; q < 4; ++q)   // K = 32 pairs per instruction
                    tc::mma_u8(tmem + g * 128, tc::desc_sw32(a0 + q * 1024, 4096, 256),
                               tc::desc_sw32(a0 + 12288 + q * 1024, 4096, 256), idesc, !(first && q == 0));
                tc::commit(&empty[s]);
                if (it % kR1Chunk == kR1Chunk - 1 || it == nt - 1) tc::commit(&dready[g]);
            }
        }
        __syncwarp();
    } else if (warp < 2 + PW) {
        // D = b + p - a for 2 x 128 rows per tile (rows of 32 bytes, 32-byte swizzle)
        const uint32_t t = threadIdx.x - 64;
        const uint32_t Pw[8] = {BZK_P0, BZK_P1, BZK_P2, BZK_P3, BZK_P4, BZK_P5, BZK_P6, BZK_P7};
        for (uint32_t it = 0; it < nt; ++it) {
            const uint32_t s = it % kR1Stages;
            tc::mbar_wait(&full[s], (it / kR1Stages) & 1);
            uint8_t *st = base + s * 24576;
#pragma unroll
            for (int e = 0; e < 8 / PW; ++e) {
                const uint32_t r = t + 32 * PW * e, m = r >> 7, j = r & 127;
                const uint32_t sw = (j >> 2) & 1, o0 = j * 32 + (sw << 4), o1 = j * 32 + ((1 - sw) << 4);
                uint8_t *tb = st + m * 12288;
                const uint4 a_lo = *reinterpret_cast<const uint4 *>(tb + o0), a_hi = *reinterpret_cast<const uint4 *>(tb + o1);
                const uint4 b_lo = *reinterpret_cast<const uint4 *>(tb + 4096 + o0),
                            b_hi = *reinterpret_cast<const uint4 *>(tb + 4096 + o1);
                const uint32_t A[8] = {a_lo.x, a_lo.y, a_lo.z, a_lo.w, a_hi.x, a_hi.y, a_hi.z, a_hi.w};
                const uint32_t Bv[8] = {b_lo.x, b_lo.y, b_lo.z, b_lo.w, b_hi.x, b_hi.y, b_hi.z, b_hi.w};
                uint32_t tp[8], d[8];
                uint64_t c = 0;
#pragma unroll
                for (int w = 0; w < 8; ++w) {   // b + p < 2^255: no carry out
                    c += (uint64_t)Bv[w] + Pw[w];
                    tp[w] = (uint32_t)c;
                    c >>= 32;
                }
                int64_t br = 0;
#pragma unroll
                for (int w = 0; w < 8; ++w) {   // (b + p) - a > 0: no borrow out
                    const int64_t v = (int64_t)tp[w] - (int64_t)A[w] + br;
                    d[w] = (uint32_t)v;
                    br = v >> 32;
                }
                *reinterpret_cast<uint4 *>(tb + 8192 + o0) = make_uint4(d[0], d[1], d[2], d[3]);
                *reinterpret_cast<uint4 *>(tb + 8192 + o1) = make_uint4(d[4], d[5], d[6], d[7]);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // D (generic writes) -> MMA reads
            tc::mbar_arrive(&prep[s]);
        }
    } else {
        const uint32_t q = warp & 3;                // TMEM lanes 32 q ..: rows of the a / b / D / unused block
                                                    // (the 4 epilogue warps cover q = 0..3 for PW = 2 or 4)
        for (uint32_t c = 0; c < nch; ++c) {
            const uint32_t g = c & 1;
            tc::mbar_wait(&dready[g], (c >> 1) & 1);
            tc::fence_after();
            if (q < 3) {
                uint32_t v[32];
                tc::ld_x32(tmem + ((q * 32) << 16) + g * 128 + q * 32, v);
                tc::wait_ld();
#pragma unroll
                for (int i = 0; i < 32; ++i) macc[i] += v[i];
            }
            tc::fence_before();
            tc::mbar_arrive(&dempty[g]);
        }
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 1) {
        tc::fence_after();
        tc::tmem_dealloc<256>(tmem);
    }
    // anti-diagonal sums s_n = sum_{i+i'=n} M[i][i'] of the three blocks, then S -> acc17 -> fe
    if (threadIdx.x < 3 * 64) s_diag[threadIdx.x >> 6][threadIdx.x & 63] = 0;
    __syncthreads();
    if (warp >= 2 + PW && (warp & 3) < 3) {
#pragma unroll
        for (int i = 0; i < 32; ++i)
            atomicAdd(&s_diag[warp & 3][lane + i], macc[i]);
    }
    __syncthreads();
    fe acc[NV];
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = fe_zero();
    if (threadIdx.x < NV && nt > 0) {
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
        // thread t holds point t's partial: 0 -> g(0), 1 -> g(1), 2 -> c_inf (Pts<2, FIRST> order)
        const fe f = acc17_to_fe(S);
#pragma unroll
        for (int t = 0; t < NV; ++t)
            if (t == (int)threadIdx.x) acc[t] = f;
    }
    round_finish<D, false>(P, b, acc, s_red, s_clu, &s_last);
}

}  // namespace bzk
