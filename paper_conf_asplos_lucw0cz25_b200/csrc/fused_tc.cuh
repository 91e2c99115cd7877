// fused_tc.cuh -- the fused fold(r_{i-1}) + eval(i) round of d = 2 BN254 proofs with the evaluation
// sums on the tensor cores (tcgen05 kind::i8); the folds stay on the integer pipe.
//
// Same round as k_round<2, ORDER, FIRST = false, TMA = true> (sumcheck.cuh: TMA-staged raw entries,
// fixed-multiplier folds written to the other ping-pong buffer), but the two summed points of
// a fused round (Pts<2, DERIVE>: t = 0 and the leading coefficient) are
//   g(0) = sum_j a0_j a1_j,   c_inf = sum_j D0_j D1_j       (a = folded entry, D = lazy b - a)
// computed as u8 products over the pairs (round1_tc.cuh header: sum_j x_j y_j = sum M[i][i'] 2^(8(i+i'))
// with M = X^T Y, K = the pairs).  Each compute warp writes its 32 pairs' (a0 | D0 | a1 | D1) bytes into
// its own 4 KiB tile (32 rows x 32 bytes per vector, 32-byte swizzle, MN-major operands) and signals
// the MMA warp, which issues one M = 128 (a0 | D0 | a1 | D1), N = 64 (a1 | D1), K = 32 product per tile
// into the CTA's TMEM accumulator; the diagonal blocks (a0 x a1, D0 x D1) are the two M's.  At most
// 32768 pairs per CTA keep every s32 entry < 32768 * 255^2 < 2^31, so one accumulator lasts the CTA.
// After the loop: anti-diagonal sums -> S (< 2^527) -> acc17_to_fe = the canonical partial k_round's
// acc17 path produces (same integers, same residue), then round_finish.
//
// This removes the two 256 x 256-bit products per pair (256 of ~910 integer-pipe slots) from the
// integer pipe, which the folds and the products shared (ncu r02c: fma-heavy 75 %, DRAM 64 %).
#pragma once
#include <stdint.h>
#include "sumcheck.cuh"
#include "tc.cuh"

namespace bzk {

constexpr int kFtCompute = 256;                    // compute threads (8 warps, as k_round)
constexpr int kFtThreads = kFtCompute + 32;        // + the MMA warp
constexpr uint64_t kFtMaxPairs = 32768;            // pairs per CTA (s32 accumulator bound)
constexpr size_t kFtSmem = 1024 + (size_t)(kFtCompute / 32) * 2 * 4096 + (size_t)(kFtCompute / 32) * 4096;

template <int ORDER>
__global__ void __launch_bounds__(kFtThreads, 2) k_fused_tc(RoundParams P, const __grid_constant__ CUtensorMap tmap) {
    constexpr int D = 2, NV = Pts<2, true>::NV;    // t = 0, inf
    using G = TmaGeo<ORDER, false>;
    static_assert(G::NSTAGE == 1 && G::SLOT == 4096, "fused-round TMA geometry");
    __shared__ fe s_red[32 * NV];
    __shared__ fe s_clu[NV];
    __shared__ int s_last;
    __shared__ __align__(8) uint64_t bars[(kFtCompute / 32) * D], tfull[kFtCompute / 32], tempty[kFtCompute / 32], dfin;
    __shared__ uint32_t s_tmem;
    __shared__ __align__(16) fe sK[8];
    extern __shared__ uint8_t ft_raw[];
    uint8_t *base = ft_raw + ((1024 - (smem_u32(ft_raw) & 1023)) & 1023);
    const uint32_t b = blockIdx.y, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t h = 1ull << P.log_h;
    const uint64_t stride = (uint64_t)P.ctas * kFtCompute;
    const fe *src = P.src + (size_t)b * D * (4 * h);
    fe *dst = P.dst + (size_t)b * D * (2 * h);
    (void)src;

    if (threadIdx.x < 8) sK[threadIdx.x] = mont_mul(P.ps[b].rmont, P.consts[kConstPow2 + threadIdx.x]);   // r 2^(32t+64)
    if (threadIdx.x == 0) {
        for (int w = 0; w < kFtCompute / 32; ++w) {
            tc::mbar_init_n(&bars[2 * w], 1);
            tc::mbar_init_n(&bars[2 * w + 1], 1);
            tc::mbar_init_n(&tfull[w], 1);
            tc::mbar_init_n(&tempty[w], 1);
        }
        tc::mbar_init_n(&dfin, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kFtCompute / 32) tc::tmem_alloc<64>(&s_tmem);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    uint8_t *tiles = base + (size_t)(kFtCompute / 32) * D * G::SLOT;   // [warp][a0 | D0 | a1 | D1][32 rows][32 B]

    if (warp < kFtCompute / 32) {
        uint8_t *wslots = base + (size_t)warp * D * G::SLOT;
        uint64_t *wbars = bars + warp * D;
        uint8_t *tile = tiles + warp * 4096;
        const uint64_t row0 = (uint64_t)b * D * (G::E * h / 4);
        const uint64_t trows = G::E * h / 4;
        const uint64_t j0 = (uint64_t)blockIdx.x * kFtCompute + warp * 32;
        if (lane == 0 && j0 < h)
#pragma unroll
            for (int m = 0; m < D; ++m)
                tma_issue<ORDER, false>(&tmap, wslots + m * G::SLOT, &wbars[m], row0 + m * trows, h, j0);
        uint32_t it = 0;
        for (uint64_t jw = j0; jw < h; jw += stride, ++it) {
            const uint64_t j = jw + lane;
            fe a[D], sv[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                uint8_t *slot = wslots + m * G::SLOT;
                mbar_wait(&wbars[m], it & 1);
                fe x[G::E];
#pragma unroll
                for (int e = 0; e < G::E; ++e) x[e] = tma_entry<ORDER, false>(slot, lane, e);
                fold_group<D, ORDER, false>(x, m, dst, h, j, sK, P.zero, a[m], sv[m]);
                __syncwarp();                  // every lane has consumed the slot
                if (lane == 0 && jw + stride < h)
                    tma_issue<ORDER, false>(&tmap, slot, &wbars[m], row0 + m * trows, h, jw + stride);
            }
            // the previous tile's product has read this warp's tile
            if (it > 0) tc::mbar_wait(&tempty[warp], (it - 1) & 1);
            const uint32_t sw = (lane >> 2) & 1, o0 = lane * 32 + (sw << 4), o1 = lane * 32 + ((1 - sw) << 4);
            auto put = [&](int v, const fe &x) {
                *reinterpret_cast<uint4 *>(tile + v * 1024 + o0) = make_uint4(x.l[0], x.l[1], x.l[2], x.l[3]);
                *reinterpret_cast<uint4 *>(tile + v * 1024 + o1) = make_uint4(x.l[4], x.l[5], x.l[6], x.l[7]);
            };
            put(0, a[0]);
            put(1, sv[0]);
            put(2, a[1]);
            put(3, sv[1]);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // tile (generic writes) -> MMA reads
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&tfull[warp]);
        }
    } else if (lane == 0) {
        // MMA warp: one product per compute-warp tile, warps visited round-robin
        const uint32_t idesc = tc::idesc_u8(128, 64, true) | (1u << 15);   // A and B MN-major
        const uint32_t tb = smem_u32(tiles);
        uint32_t nw[kFtCompute / 32], nmax = 0;
#pragma unroll
        for (int w = 0; w < kFtCompute / 32; ++w) {
            const uint64_t j0 = (uint64_t)blockIdx.x * kFtCompute + w * 32;
            nw[w] = j0 < h ? (uint32_t)((h - 1 - j0) / stride + 1) : 0;
            nmax = nw[w] > nmax ? nw[w] : nmax;
        }
        bool first = true;
        for (uint32_t it = 0; it < nmax; ++it) {
#pragma unroll
            for (int w = 0; w < kFtCompute / 32; ++w) {
                if (it >= nw[w]) continue;
                tc::mbar_wait(&tfull[w], it & 1);
                tc::fence_after();
                const uint32_t t0 = tb + w * 4096;
                tc::mma_u8(tmem, tc::desc_sw32(t0, 1024, 256), tc::desc_sw32(t0 + 2048, 1024, 256), idesc, !first);
                first = false;
                tc::commit(&tempty[w]);
            }
        }
        if (nmax > 0) tc::commit(&dfin);
    }
    __syncwarp();
    // anti-diagonal sums of the two diagonal blocks (warps 0 and 1 read TMEM lanes 0..31 / 32..63)
    uint32_t *sM = reinterpret_cast<uint32_t *>(base);   // [2][32][33] (reuses the TMA slots)
    __shared__ unsigned long long s_diag[2][64];
    const bool any = (uint64_t)blockIdx.x * kFtCompute < h;
    tc::fence_before();
    __syncthreads();
    if (warp < 2 && any) {
        tc::mbar_wait(&dfin, 0);
        tc::fence_after();
        uint32_t v[32];
        tc::ld_x32(tmem + ((warp * 32) << 16) + warp * 32, v);
        tc::wait_ld();
#pragma unroll
        for (int i = 0; i < 32; ++i) sM[(warp * 32 + lane) * 33 + i] = v[i];   // row = byte `lane` of a0 / D0
    }
    tc::fence_before();
    __syncthreads();
    if (warp == kFtCompute / 32) {
        tc::fence_after();
        tc::tmem_dealloc<64>(tmem);
    }
    if (threadIdx.x < 128) {
        const uint32_t t = threadIdx.x >> 6, n = threadIdx.x & 63;
        unsigned long long s = 0;
        if (any)
            for (int i = 0; i < 32; ++i)
                if (n >= (uint32_t)i && n - i < 32) s += sM[(t * 32 + i) * 33 + (n - i)];
        s_diag[t][n] = s;
    }
    __syncthreads();
    fe acc[NV];
#pragma unroll
    for (int t = 0; t < NV; ++t) acc[t] = fe_zero();
    if (threadIdx.x < NV && any) {
        acc17 S = acc17_zero();
        for (int n = 0; n < 63; ++n) {   // add s_n 2^(8n) (s_n < 2^36)
            const unsigned long long v = s_diag[threadIdx.x][n];
            const int w0 = (8 * n) >> 5, sh = (8 * n) & 31;
            uint64_t cur = (uint64_t)S.w[w0] + (uint32_t)(v << sh);
            S.w[w0] = (uint32_t)cur;
            uint64_t carry = (cur >> 32) + (sh ? (v >> (32 - sh)) : (v >> 32));
            for (int w = w0 + 1; w < 17 && carry; ++w) {
                cur = (uint64_t)S.w[w] + (uint32_t)carry;
                S.w[w] = (uint32_t)cur;
                carry = (carry >> 32) + (cur >> 32);
            }
        }
        const fe f = acc17_to_fe(S);   // thread 0: g(0) partial, thread 1: c_inf partial
#pragma unroll
        for (int t = 0; t < NV; ++t)
            if (t == (int)threadIdx.x) acc[t] = f;
    }
    round_finish<D, true>(P, b, acc, s_red, s_clu, &s_last);
}

}  // namespace bzk
