// fused_tc.cuh -- sum-check rounds with the evaluation sums on the tensor cores (tcgen05 kind::i8);
// the folds and the first d - 2 products of every point stay on the integer pipe.
//
// Same rounds as k_round<D, ORDER, FIRST, TMA = true> (sumcheck.cuh: TMA-staged raw entries,
// fixed-multiplier folds written to the other ping-pong buffer), but the LAST product of every
// summed point -- eval_one's mul_acc(acc_t, X_t, Y_t), a 256 x 256-bit product added unreduced into a
// 544-bit accumulator -- is a sum over the pairs sum_j X_t(j) Y_t(j) computed as u8 products
// (round1_tc.cuh header: sum_j x_j y_j = sum M[i][i'] 2^(8(i+i')) with M = X^T Y, K = the pairs):
//   d = 2 fused rounds (points 0, inf):      X = a0 | D0,            Y = a1 | D1       (a = folded entry,
//                                                                                       D = lazy b - a)
//   d = 3 fused rounds (points 0, 2, inf):   X_t = x0(t) x1(t) R^-1, Y_t = x2(t)
//   d = 3 round 1 (points 0, 1, 2, inf):     same, x_m(t) from the raw (a, b)
// Each compute warp writes its 32 pairs' operand bytes into its own tile (32 rows x 32 bytes per vector,
// 32-byte swizzle, MN-major operands; FtGeo) and signals the MMA warp, which issues one M = 128, N = 32 NV
// (d = 2: 64), K = 32 product per tile into the CTA's TMEM accumulator; the diagonal blocks are the M_t.
// At most 32768 pairs per CTA keep every s32 entry < 32768 * 255^2 < 2^31, so one accumulator lasts the
// CTA.  After the loop: anti-diagonal sums -> S (< 2^527) -> acc17_to_fe = the canonical partial
// k_round's acc17 path produces (same integers, same residue), then round_finish.
//
// d = 2 removes the two 256 x 256-bit products per pair (256 of ~910 integer-pipe slots) from the
// integer pipe, which the folds and the products shared (ncu r02c: fma-heavy 75 %, DRAM 64 %); d = 3
// removes NV of its 2 NV products per pair (the Montgomery products x0 x1 stay on the integer pipe).
#pragma once
#include <stdint.h>
#include "sumcheck.cuh"
#include "tc.cuh"

namespace bzk {

// compute warps per CTA: 8 for d = 2 (two CTAs per SM); d = 3 (one CTA per SM by shared memory, long
// integer-pipe chains per pair: 6 folds + 3 Montgomery products, or round 1's 4 Montgomery products)
// runs 12 for latency hiding.  One TMA slot per (warp, table): the copy of the warp's next tile is issued
// as soon as every lane has consumed the slot, so it lands while the rest of the iteration computes.
// The small late fused rounds of d = 2 (h <= 2^12 pairs per proof: a few microseconds of work per CTA,
// dominated by the CTA's fixed costs and the proof's serial finalisation) run NW = 2: one CTA of 96
// threads per proof (two above 2^11), 7 resident per SM (registers), so a 1024-proof wave is one
// CTA wave instead of several.
template <int D, bool FIRST> __host__ __device__ constexpr int ft_nw() { return D == 3 ? (FIRST ? 12 : 10) : 8; }
constexpr int kFtSmallNW = 2;
__host__ __device__ constexpr int ft_threads(int nw) { return 32 * nw + 32; }   // + the MMA warp
__host__ __device__ constexpr int ft_minb(int D, int nw) { return D == 3 ? 1 : nw == kFtSmallNW ? 7 : 2; }
constexpr uint64_t kFtMaxPairs = 32768;            // pairs per CTA (s32 accumulator bound)

// Per-warp operand tile of one MMA (32 pairs = K), MN-major 32-byte rows, 1 KiB per vector:
//   d = 2 fused:   A = (a0 | D0 | a1 | D1) M = 128, B = (a1 | D1) at +2 KiB, N = 64   (points 0, inf)
//   d = 3 fused:   A = (X0 | X2 | Xinf | Y0), B = (Y0 | Y2 | Yinf) at +3 KiB, N = 96 (points 0, 2, inf)
//   d = 3 round 1: A = (X0 | X1 | X2 | Xinf), B = (Y0 | Y1 | Y2 | Yinf) at +4 KiB, N = 128
// with X_t = x0(t) x1(t) R^-1 (the lazy Montgomery product eval_one forms, < 2p) and Y_t = x2(t) (lazy,
// < 2p): eval_one's mul_acc(acc_t, X_t, Y_t) summed on the tensor cores.  Diagonal block t (rows 32t,
// columns 32t) of D is M_t = X_t^T Y_t.  Rows 96..127 of the d = 3 fused A overlap B's first
// vector (those D rows are never read).
template <int D, bool FIRST> struct FtGeo;
template <> struct FtGeo<2, false> { static constexpr uint32_t TILE = 4096, BOFF = 2048, N = 64, TCOLS = 64; };
// d = 3 fused rounds (wide): vectors 0..5 = X0 lo|hi, X2 lo|hi, Xinf lo|hi, 6..8 = Y0, Y2, Yinf; MMAs
// (X0, X2) x (Y0 | Y2) (N = 64) and (Xinf, -) x Yinf (N = 32)
template <> struct FtGeo<3, false> { static constexpr uint32_t TILE = 9216, BOFF = 6144, N = 64, TCOLS = 128; };
// d = 3 round 1 ("wide"): X_t = x0(t) x1(t) UNREDUCED (512 bits = two 32-byte vectors, lo | hi), so the
// integer pipe does 64 limb products per point instead of a Montgomery product's 136; vectors
// 0..7 = X0 lo|hi, X1 lo|hi, X2 lo|hi, Xinf lo|hi, 8..11 = Y0, Y1, Y2, Yinf.  Two MMAs per tile into two
// 64-column TMEM accumulators: (X0, X1) x (Y0 | Y1) and (X2, Xinf) x (Y2 | Yinf).
template <> struct FtGeo<3, true> { static constexpr uint32_t TILE = 12288, BOFF = 8192, N = 64, TCOLS = 128; };

template <int D, bool FIRST, int NW = ft_nw<D, FIRST>()>
constexpr size_t ft_smem() {
    return 1024 + (size_t)NW * D * TmaGeo<0, FIRST>::SLOT + (size_t)NW * FtGeo<D, FIRST>::TILE;
}

// d = 3: table m's value at summed point idx (Pts<3, DERIVE> order), exactly as eval_one forms it
// (a = entry / folded entry, s = b (round 1) or the lazy delta (fused rounds), dl = round 1's delta)
template <bool DERIVE>
__device__ __forceinline__ fe d3_point(const fe &a, const fe &s, const fe &dl, int idx) {
    const int t = point_t<3, DERIVE>(idx);
    if (t == 0) return a;
    if (t == 1) return s;
    if (t < 0) return DERIVE ? s : dl;
    // t == 2
    if (DERIVE) return lz_red(lz_add(lz_red(lz_add(a, s)), s));
    return lz_red(lz_add(s, dl));
}

template <int D, int ORDER, bool FIRST, int NW>
__global__ void __launch_bounds__(ft_threads(NW), ft_minb(D, NW)) k_fused_tc(RoundParams P, const __grid_constant__ CUtensorMap tmap) {
    static_assert(D == 2 ? !FIRST : D == 3, "k_fused_tc shapes: d = 2 fused rounds, d = 3 round 1 and fused rounds");
    static_assert(NW >= Pts<D, !FIRST>::NV, "the epilogue reads one TMEM block per compute warp");
    constexpr bool DERIVE = !FIRST;
    constexpr int NV = Pts<D, DERIVE>::NV;
    using G = TmaGeo<ORDER, FIRST>;
    using FG = FtGeo<D, FIRST>;
    constexpr int NS = 1, kFtCompute = 32 * NW;
    __shared__ fe s_red[32 * NV];
    __shared__ fe s_clu[NV];
    __shared__ int s_last;
    __shared__ __align__(8) uint64_t bars[NW * D * NS], tfull[NW], tempty[NW], dfin;
    __shared__ uint32_t s_tmem;
    __shared__ __align__(16) fe sK[8];
    extern __shared__ uint8_t ft_raw[];
    uint8_t *base = ft_raw + ((1024 - (smem_u32(ft_raw) & 1023)) & 1023);
    BZK_ASSERT((size_t)(base - ft_raw) + (size_t)NW * (D * G::SLOT + FG::TILE) <= dyn_smem_bytes() &&
               (size_t)(D == 3 ? 2 * NV : NV) * 32 * 33 * 4 <= (size_t)NW * D * G::SLOT);
    const uint32_t b = blockIdx.y, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint64_t h = 1ull << P.log_h;
    const uint64_t stride = (uint64_t)P.ctas * kFtCompute;
    fe *dst = FIRST ? nullptr : P.dst + (size_t)b * D * (2 * h);

    if (!FIRST && threadIdx.x < 8)
        sK[threadIdx.x] = mont_mul(P.ps[b].rmont, P.consts[kConstPow2 + threadIdx.x]);   // r 2^(32t+64)
    if (threadIdx.x == 0) {
        for (int q = 0; q < NW * D * NS; ++q) tc::mbar_init_n(&bars[q], 1);
        for (int w = 0; w < NW; ++w) {
            tc::mbar_init_n(&tfull[w], 1);
            tc::mbar_init_n(&tempty[w], 1);
        }
        tc::mbar_init_n(&dfin, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == NW) tc::tmem_alloc<FG::TCOLS>(&s_tmem);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    uint8_t *tiles = base + (size_t)NW * D * NS * G::SLOT;   // [warp][vectors][32 rows][32 B]

    if (warp < NW) {
        uint8_t *wslots = base + (size_t)warp * D * NS * G::SLOT;
        uint64_t *wbars = bars + warp * D * NS;
        uint8_t *tile = tiles + warp * FG::TILE;
        const uint64_t row0 = (uint64_t)b * D * (G::E * h / 4);
        const uint64_t trows = G::E * h / 4;
        const uint64_t j0 = (uint64_t)blockIdx.x * kFtCompute + warp * 32;
        if (lane == 0 && j0 < h)
#pragma unroll
            for (int m = 0; m < D; ++m)
                tma_issue<ORDER, FIRST>(&tmap, wslots + m * G::SLOT, &wbars[m], row0 + m * trows, h, j0);
        const uint32_t sw = (lane >> 2) & 1, o0 = lane * 32 + (sw << 4), o1 = lane * 32 + ((1 - sw) << 4);
        auto put = [&](int v, const fe &x) {
            BZK_ASSERT((uint32_t)v * 1024 + 1024 <= FG::TILE);
            *reinterpret_cast<uint4 *>(tile + v * 1024 + o0) = make_uint4(x.l[0], x.l[1], x.l[2], x.l[3]);
            *reinterpret_cast<uint4 *>(tile + v * 1024 + o1) = make_uint4(x.l[4], x.l[5], x.l[6], x.l[7]);
        };
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
                for (int e = 0; e < G::E; ++e) x[e] = tma_entry<ORDER, FIRST>(slot, lane, e);
                fold_group<D, ORDER, FIRST, D == 2>(x, m, dst, h, j, sK, P.zero, a[m], sv[m]);
                __syncwarp();                  // every lane has consumed the slot
                if (lane == 0 && jw + stride < h)
                    tma_issue<ORDER, FIRST>(&tmap, slot, &wbars[m], row0 + m * trows, h, jw + stride);
            }
            // the previous tile's product has read this warp's tile
            if (it > 0) tc::mbar_wait(&tempty[warp], (it - 1) & 1);
            if constexpr (D == 2) {
                put(0, a[0]);
                put(1, sv[0]);
                put(2, a[1]);
                put(3, sv[1]);
            } else {
                fe dl[D];
#pragma unroll
                for (int m = 0; m < D; ++m) dl[m] = FIRST ? lz_red(lz_sub(sv[m], a[m])) : sv[m];
                if constexpr (FIRST) {
                    // x0(t) x1(t) is a quadratic in t, so X_2 = 2 X_1 + 2 X_inf - X_0 (+ 4p^2, a multiple of p
                    // that keeps it non-negative): the same residue as x0(2) x1(2) with 3 products per pair.
                    // Bounds: x_m(t) < 2p, so X_t < 4p^2 and X_2 < 14p^2 < 2^512.
                    const uint32_t P4[16] = {0x80000004u, 0x230fac9fu, 0x72cd0000u, 0x1fc9888fu, 0xa326edffu,
                                             0xffa698b1u, 0xa08776c3u, 0x9b3865d7u, 0x1ed8bf9eu, 0xb1dd49edu,
                                             0x4de74f7cu, 0x17dceec3u, 0x0d234872u, 0x6669bdf0u, 0xd8f2fe71u,
                                             0x249712e1u};   // 4 p^2
                    uint32_t X2[16];
#pragma unroll
                    for (int idx = 0; idx < NV; ++idx) {
                        put(8 + idx, d3_point<DERIVE>(a[2], sv[2], dl[2], idx));
                        if (idx == 2) continue;
                        acc17 W = acc17_zero();
                        mul_acc(W, d3_point<DERIVE>(a[0], sv[0], dl[0], idx), d3_point<DERIVE>(a[1], sv[1], dl[1], idx));
                        fe lo, hi;
#pragma unroll
                        for (int q = 0; q < 8; ++q) { lo.l[q] = W.w[q]; hi.l[q] = W.w[8 + q]; }
                        put(2 * idx, lo);
                        put(2 * idx + 1, hi);
                        if (idx == 0) {   // X2 = 4p^2 - X0
                            int64_t br = 0;
#pragma unroll
                            for (int q = 0; q < 16; ++q) {
                                const int64_t v = (int64_t)P4[q] - (int64_t)W.w[q] + br;
                                X2[q] = (uint32_t)v;
                                br = v >> 32;
                            }
                        } else {          // X2 += 2 X_1, 2 X_inf
                            uint64_t c = 0;
#pragma unroll
                            for (int q = 0; q < 16; ++q) {
                                c += (uint64_t)X2[q] + 2ull * W.w[q];
                                X2[q] = (uint32_t)c;
                                c >>= 32;
                            }
                        }
                    }
                    fe lo, hi;
#pragma unroll
                    for (int q = 0; q < 8; ++q) { lo.l[q] = X2[q]; hi.l[q] = X2[8 + q]; }
                    put(4, lo);
                    put(5, hi);
                } else {   // points 0, 2, inf: X_t = x0(t) x1(t) unreduced (x_m(t) < 2p: X_t < 4p^2 < 2^512)
#pragma unroll
                    for (int idx = 0; idx < NV; ++idx) {
                        acc17 W = acc17_zero();
                        mul_acc(W, d3_point<DERIVE>(a[0], sv[0], dl[0], idx), d3_point<DERIVE>(a[1], sv[1], dl[1], idx));
                        fe lo, hi;
#pragma unroll
                        for (int q = 0; q < 8; ++q) { lo.l[q] = W.w[q]; hi.l[q] = W.w[8 + q]; }
                        put(2 * idx, lo);
                        put(2 * idx + 1, hi);
                        put(6 + idx, d3_point<DERIVE>(a[2], sv[2], dl[2], idx));
                    }
                }
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // tile (generic writes) -> MMA reads
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&tfull[warp]);
        }
    } else if (lane == 0) {
        // MMA warp: one product per compute-warp tile, issued for whichever warp's tile is ready (a fixed
        // round-robin order would hold every warp to the slowest one: each has a single tile)
        const uint32_t idesc = tc::idesc_u8(128, FG::N, true) | (1u << 15);   // A and B MN-major
        const uint32_t tb = smem_u32(tiles);
        uint32_t nw[NW], done[NW], left = 0, nmax = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            const uint64_t j0 = (uint64_t)blockIdx.x * kFtCompute + w * 32;
            nw[w] = j0 < h ? (uint32_t)((h - 1 - j0) / stride + 1) : 0;
            done[w] = 0;
            left += nw[w];
            nmax = nw[w] > nmax ? nw[w] : nmax;
        }
        bool first = true;
        while (left) {
            bool issued = false;
#pragma unroll
            for (int w = 0; w < NW; ++w) {
                if (done[w] < nw[w] && tc::mbar_test(&tfull[w], done[w] & 1)) {
                    tc::fence_after();
                    const uint32_t t0 = tb + w * FG::TILE;
                    if constexpr (D == 3 && FIRST) {   // (X0 | X1) x (Y0 | Y1), (X2 | Xinf) x (Y2 | Yinf)
                        tc::mma_u8(tmem, tc::desc_sw32(t0, 1024, 256), tc::desc_sw32(t0 + 8192, 1024, 256), idesc, !first);
                        tc::mma_u8(tmem + 64, tc::desc_sw32(t0 + 4096, 1024, 256), tc::desc_sw32(t0 + 10240, 1024, 256),
                                   idesc, !first);
                    } else if constexpr (D == 3) {     // (X0 | X2) x (Y0 | Y2), (Xinf | -) x Yinf
                        const uint32_t idesc32 = tc::idesc_u8(128, 32, true) | (1u << 15);
                        tc::mma_u8(tmem, tc::desc_sw32(t0, 1024, 256), tc::desc_sw32(t0 + 6144, 1024, 256), idesc, !first);
                        tc::mma_u8(tmem + 64, tc::desc_sw32(t0 + 4096, 1024, 256), tc::desc_sw32(t0 + 8192, 1024, 256),
                                   idesc32, !first);
                    } else {
                        tc::mma_u8(tmem, tc::desc_sw32(t0, 1024, 256), tc::desc_sw32(t0 + FG::BOFF, 1024, 256), idesc,
                                   !first);
                    }
                    first = false;
                    tc::commit(&tempty[w]);
                    ++done[w];
                    --left;
                    issued = true;
                }
            }
            if (!issued) __nanosleep(100);   // a tile takes microseconds to build: keep this warp off the issue slots
        }
        if (nmax > 0) tc::commit(&dfin);
    }
    __syncwarp();
    // anti-diagonal sums of the diagonal blocks (warp t reads TMEM lanes 32t.., columns 32t..; the wide
    // d = 3 round 1 has NB = 8 blocks: warp q reads its quadrant of both accumulators)
    constexpr bool WIDE = D == 3;
    constexpr int NB = WIDE ? 2 * NV : NV;
    uint32_t *sM = reinterpret_cast<uint32_t *>(base);   // [NB][32][33] (reuses the TMA slots)
    __shared__ unsigned long long s_diag[NB][64];
    const bool any = (uint64_t)blockIdx.x * kFtCompute < h;
    tc::fence_before();
    __syncthreads();
    if (warp < (uint32_t)(WIDE ? 4 : NV) && any) {
        tc::mbar_wait(&dfin, 0);
        tc::fence_after();
#pragma unroll
        for (int g = 0; g < (WIDE ? 2 : 1); ++g) {
            if (WIDE && !FIRST && g == 1 && warp >= 2) break;   // (Xinf | -) x Yinf: lanes 0..63 only
            uint32_t v[32];
            const uint32_t col = WIDE ? g * 64 + (warp >> 1) * 32 : warp * 32;
            tc::ld_x32(tmem + ((warp * 32) << 16) + col, v);
            tc::wait_ld();
            const uint32_t blk = WIDE ? g * 4 + warp : warp;
#pragma unroll
            for (int i = 0; i < 32; ++i) sM[(blk * 32 + lane) * 33 + i] = v[i];   // row = byte `lane` of X_t
        }
    }
    tc::fence_before();
    __syncthreads();
    if (warp == NW) {
        tc::fence_after();
        tc::tmem_dealloc<FG::TCOLS>(tmem);
    }
    for (uint32_t q = threadIdx.x; q < NB * 64; q += blockDim.x) {   // NW = 2: fewer threads than sums
        const uint32_t t = q >> 6, n = q & 63;
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
        fe f;
        if constexpr (WIDE) {
            // S_t = sum_j X_t Y_t = B_lo + 2^256 B_hi (< 2^788, 25 words); partial = S_t R^-2 mod p (the
            // Montgomery products of the narrow path carried one R^-1 each): 16 REDC word steps
            const uint32_t Pw[8] = {BZK_P0, BZK_P1, BZK_P2, BZK_P3, BZK_P4, BZK_P5, BZK_P6, BZK_P7};
            uint32_t T[26];
            for (int q = 0; q < 26; ++q) T[q] = 0;
            for (int half = 0; half < 2; ++half)
                for (int n = 0; n < 63; ++n) {   // add s_n 2^(8n + 256 half) (s_n < 2^36)
                    const unsigned long long v = s_diag[2 * threadIdx.x + half][n];
                    const int w0 = ((8 * n) >> 5) + 8 * half, sh = (8 * n) & 31;
                    uint64_t cur = (uint64_t)T[w0] + (uint32_t)(v << sh);
                    T[w0] = (uint32_t)cur;
                    uint64_t carry = (cur >> 32) + (sh ? (v >> (32 - sh)) : (v >> 32));
                    for (int w = w0 + 1; w < 26 && carry; ++w) {
                        cur = (uint64_t)T[w] + (uint32_t)carry;
                        T[w] = (uint32_t)cur;
                        carry = (carry >> 32) + (cur >> 32);
                    }
                }
            for (int i = 0; i < 16; ++i) {   // T += m p 2^(32 i) clears word i
                const uint32_t m = T[i] * BZK_NP0;
                uint64_t c = 0;
                for (int j = 0; j < 8; ++j) {
                    const uint64_t x = (uint64_t)m * Pw[j] + T[i + j] + c;
                    T[i + j] = (uint32_t)x;
                    c = x >> 32;
                }
                for (int j = i + 8; j < 26 && c; ++j) {
                    const uint64_t x = (uint64_t)T[j] + c;
                    T[j] = (uint32_t)x;
                    c = x >> 32;
                }
            }
            // W = T[16..25] = (S + q p) / 2^512 < 2^272 + p:  W = lo + hi 2^256,  hi 2^256 = mont_mul(hi, R^2)
            fe lo, hi = fe_zero();
            for (int q = 0; q < 8; ++q) lo.l[q] = T[16 + q];
            hi.l[0] = T[24];
            hi.l[1] = T[25];
            f = fe_add(fe_reduce_256(lo), mont_mul(hi, fe_const(2)));
        } else {
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
            f = acc17_to_fe(S);   // thread t: point t's partial (Pts<D, DERIVE> order)
        }
#pragma unroll
        for (int t = 0; t < NV; ++t)
            if (t == (int)threadIdx.x) acc[t] = f;
    }
    round_finish<D, DERIVE>(P, b, acc, s_red, s_clu, &s_last);
}

}  // namespace bzk
