// encoder.cuh -- batched linear-time (Spielman-style) encoding on B200 (
// DESIGN.md readings R21-R24).
//
// P:113-117 (Sec. 2.4, Fig. 3): stage l multiplies its input x_l by the first graph's sparse matrix
// A_l, the result is encoded by the next stage, and the returned vector z is multiplied by the second
// graph's matrix B_l; the stage outputs x_l || z || B_l z.  The base stage outputs x_L || G0 x_L.
// As the paper does (Fig. 6) the recursion is unrolled into two launch chains: forward
// y_{l+1} = A_l y_l for l = 0..L-1, the base product, then B_l products in reverse (small to large).
// Every product is written straight into its place in the codeword, so the whole encoding runs in
// place in the caller's [B][2n] buffer:  c_l = (x_l | c_{l+1} | w_l) at offset o_l, o_{l+1} = o_l + n_l.
//
// The sparse matrix-vector kernel (B200-first, not the paper's per-thread rows with bucket-sorted
// warps, though it keeps their length sort): the matrix is stored as SELL-32 -- rows sorted
// by length (descending), 32 rows per warp slice, entries interleaved so lane i of slice s reads
// entry t at off_s + 32 t + i (coalesced 256-bit loads of the weights, 32-bit loads of the columns).
// One thread computes its row for K codewords of the batch, sharing every weight load; each sum
// is accumulated UNREDUCED (512-bit products in a 544-bit accumulator, 64 limb products per edge)
// and reduced once.  Weights are stored in Montgomery form (w R), so the reduction's R^{-1}
// yields the plain sum.  CTAs walk all slices of one codeword group before the next, so the
// group's source vectors stay resident in the 126 MB L2 while the weights stream (evict-first).
#pragma once
#include <stdint.h>
#include "field.cuh"
#include "sumcheck.cuh"

namespace bzk {
namespace enc {

struct SpmvParams {
    const uint32_t *perm;       // [slices * 32] original row of each (slice, lane); 0xffffffff = padding
    const uint64_t *slice_off;  // [slices] first entry of the slice
    const uint32_t *slice_w;    // [slices] entries per row in the slice (the slice's longest row)
    const uint32_t *col;        // [entries] left vertex (index into the source vector)
    const fe *val;              // [entries] weight * R mod p (padding: 0)
    uint32_t slices;
    const fe *src;              // source vector of codeword 0; codeword b at src + b * stride
    fe *dst;                    // destination vector of codeword 0
    uint64_t stride;            // elements per codeword (2n)
    uint64_t batch;             // codewords
};

#ifndef BZK_ENC_K
#define BZK_ENC_K 2      // codewords per thread (share every weight load)
#endif
#ifndef BZK_ENC_U
#define BZK_ENC_U 2      // entries per loop iteration (their gathers are in flight together)
#endif

// Gathers carry an L2 evict_last policy and the weight stream evict_first, so the streamed weights
// do not push the live source vectors out of L2 (+1-3 % on B200).

__device__ __forceinline__ uint64_t l2_policy_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t l2_policy_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ fe ld_fe_hint(const fe *p, uint64_t pol) {
    fe r;
    asm("ld.global.nc.L2::cache_hint.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8], %9;"
        : "=r"(r.l[0]), "=r"(r.l[1]), "=r"(r.l[2]), "=r"(r.l[3]), "=r"(r.l[4]), "=r"(r.l[5]), "=r"(r.l[6]),
          "=r"(r.l[7])
        : "l"(p), "l"(pol));
    return r;
}
#define BZK_ENC_GATHER(x, ptr) (x) = ld_fe_hint((ptr), pol_last)
#define BZK_ENC_WEIGHT(ptr) ld_fe_hint((ptr), pol_first)

#ifndef BZK_ENC_TPB
#define BZK_ENC_TPB 128  // threads per CTA (4 warp slices; finer occupancy steps at ~100 registers)
#endif

// minBlocks = 1 in the launch bounds is not a no-op: ptxas then allocates 120 registers (4 CTAs/SM)
// instead of 100 (5 CTAs/SM), and the 120-register schedule is 9 % faster on B200 (enc20 75.8 vs
// 82.5 ms per step, profiles/r01l_bench_enc20.json vs r02/bench_enc20_r02z.json)
template <int K, int U>
__global__ void __launch_bounds__(BZK_ENC_TPB, 1) k_spmv(SpmvParams p) {
    const uint32_t lane = threadIdx.x & 31;
    constexpr uint32_t SPC = BZK_ENC_TPB / 32;   // slices per CTA
    const uint32_t warp = threadIdx.x >> 5;
    const uint32_t slice = blockIdx.x * SPC + warp;
    if (slice >= p.slices) return;
    const uint64_t b0 = (uint64_t)blockIdx.y * K;
    if (b0 >= p.batch) return;
    const uint32_t row = p.perm[(size_t)slice * 32 + lane];
    const uint32_t W = p.slice_w[slice];
    const uint64_t off = p.slice_off[slice] + lane;
    const uint64_t pol_last = l2_policy_last(), pol_first = l2_policy_first();
    acc17 acc[K];
#pragma unroll
    for (int q = 0; q < K; ++q) acc[q] = acc17_zero();
    const fe *src[K];
#pragma unroll
    for (int q = 0; q < K; ++q) src[q] = p.src + (b0 + q < p.batch ? b0 + q : b0) * p.stride;
    uint32_t t = 0;
#pragma unroll 1
    for (; U > 1 && t + U <= W; t += U) {
        uint32_t c[U];
        fe w[U], x[U][K];
#pragma unroll
        for (int u = 0; u < U; ++u) c[u] = __ldg(p.col + off + (uint64_t)(t + u) * 32);
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int q = 0; q < K; ++q) BZK_ENC_GATHER(x[u][q], src[q] + c[u]);
#pragma unroll
        for (int u = 0; u < U; ++u) w[u] = BZK_ENC_WEIGHT(p.val + off + (uint64_t)(t + u) * 32);
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int q = 0; q < K; ++q) mul_acc(acc[q], w[u], x[u][q]);
    }
#pragma unroll 1
    for (; t < W; ++t) {
        const uint64_t e = off + (uint64_t)t * 32;
        const uint32_t c = __ldg(p.col + e);
        const fe w = BZK_ENC_WEIGHT(p.val + e);
#pragma unroll
        for (int q = 0; q < K; ++q) {
            fe x;
            BZK_ENC_GATHER(x, src[q] + c);
            mul_acc(acc[q], w, x);
        }
    }
    if (row == 0xffffffffu) return;
#pragma unroll
    for (int q = 0; q < K; ++q)
        if (b0 + q < p.batch) st_fe(p.dst + (b0 + q) * p.stride + row, acc17_to_fe(acc[q]));
}

// weights -> Montgomery form (w * R mod p), in place
static __global__ void k_to_mont(fe *v, uint64_t n) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        st_fe(v + i, mont_mul(ld_fe(v + i), fe_const(2)));
}

}  // namespace enc

// k_enc.cu
cudaError_t enc_launch_spmv(dim3 grid, uint32_t threads, cudaStream_t s, const enc::SpmvParams &p);
cudaError_t enc_launch_to_mont(fe *v, uint64_t n, cudaStream_t s);

}  // namespace bzk
