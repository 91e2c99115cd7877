// gl.cuh -- the batched sum-check prover over the Goldilocks field p = 2^64 - 2^32 + 1
// (reading R15): one 8-byte word per element, so a degree-2 round
// moves 4x fewer bytes per product than BN254 and the path becomes HBM-bound -- the regime of the
// north star's "achieved HBM GB/s against about 8 TB/s for the memory-bound low-degree case".
//
// Same method as sumcheck.cuh (Alg. 1 generalised; rows a2-a7): round 1 evaluates,
// rounds 2.. fuse fold(r_{i-1}) with eval(i) through ping-pong buffers, one kernel per round
// with a last-CTA ticket that reduces, hashes (SHA-256) and publishes r_i, then an on-chip
// tail.  Arithmetic is cheap here, so every point t = 0..d is summed directly; the kernel's job is
// to stream: 16-byte vector loads, several pairs in flight per thread.
#pragma once
#include <stdint.h>
#include "sha256.cuh"

namespace bzk {
namespace gl {

constexpr uint64_t P = 0xffffffff00000001ull;
constexpr uint64_t EPS = 0xffffffffull;   // 2^64 mod p

__device__ __forceinline__ uint64_t add(uint64_t a, uint64_t b) {   // canonical in/out
    uint64_t s = a + b;
    if (s < a) s += EPS;          // a + b - 2^64 + (2^64 mod p) = a + b - p  (< p)
    else if (s >= P) s -= P;
    return s;
}
__device__ __forceinline__ uint64_t sub(uint64_t a, uint64_t b) {   // canonical in/out
    uint64_t d = a - b;
    if (a < b) d -= EPS;          // a - b + 2^64 - (2^64 - p)
    return d;
}
// x = hi 2^64 + lo -> x mod p, using 2^64 = 2^32 - 1 and 2^96 = -1 (mod p)
__device__ __forceinline__ uint64_t reduce128(uint64_t hi, uint64_t lo) {
    const uint64_t hh = hi >> 32, hl = hi & EPS;
    uint64_t t0 = lo - hh;
    if (lo < hh) t0 -= EPS;
    const uint64_t t1 = (hl << 32) - hl;
    uint64_t t2 = t0 + t1;
    if (t2 < t1) t2 += EPS;
    return t2 >= P ? t2 - P : t2;
}
__device__ __forceinline__ uint64_t mul(uint64_t a, uint64_t b) { return reduce128(__umul64hi(a, b), a * b); }

struct State {
    uint32_t st[8];   // transcript state_i
    uint64_t r;       // r_i (canonical)
    uint64_t pad;
};

struct RoundParams {
    const uint64_t *src;   // FIRST: [Bw][D][2h]; else [Bw][D][4h]
    uint64_t *dst;         // !FIRST: [Bw][D][2h]
    uint32_t log_h, round, k, order, ctas, given;
    uint64_t *partials;    // [Bw][ctas][D+1]
    uint32_t *tickets;     // [Bw]
    State *ps;             // [Bw]
    uint64_t *round_evals; // [Bw][k][D+1]
    uint64_t *challenges;  // [Bw][k]
    uint64_t *claims;      // [Bw] (may be null)
};

struct TailParams {
    const uint64_t *src;
    uint32_t log_h0, i0, k, order, given;
    State *ps;
    uint64_t *round_evals, *challenges, *final_evals, *claims;
};

template <int V>
__device__ __forceinline__ void block_reduce(uint64_t (&acc)[V], uint64_t *smem) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = (blockDim.x + 31) >> 5;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = add(acc[v], __shfl_down_sync(0xffffffffu, acc[v], off));
    if (lane == 0)
#pragma unroll
        for (int v = 0; v < V; ++v) smem[warp * V + v] = acc[v];
    __syncthreads();
    if (warp == 0) {
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = lane < nwarps ? smem[lane * V + v] : 0ull;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1)
#pragma unroll
            for (int v = 0; v < V; ++v) acc[v] = add(acc[v], __shfl_down_sync(0xffffffffu, acc[v], off));
    }
    __syncthreads();
}

// g(t) for t = 0..D of one pair, accumulated
template <int D>
__device__ __forceinline__ void eval_pair(const uint64_t (&a)[D], const uint64_t (&b)[D], uint64_t (&acc)[D + 1]) {
    uint64_t v[D], dl[D];
#pragma unroll
    for (int m = 0; m < D; ++m) { v[m] = a[m]; dl[m] = sub(b[m], a[m]); }
#pragma unroll
    for (int t = 0; t <= D; ++t) {
        if (t) {
#pragma unroll
            for (int m = 0; m < D; ++m) v[m] = add(v[m], dl[m]);
        }
        uint64_t prod = v[0];
#pragma unroll
        for (int m = 1; m < D; ++m) prod = mul(prod, v[m]);
        acc[t] = add(acc[t], prod);
    }
}

// Lazy evaluation sums: the last product of every point is accumulated
// unreduced into a 192-bit accumulator (lo, hi, top) and reduced once per thread, instead of a
// 128 -> 64-bit reduction plus a canonical addition per product (the round kernels were ALU-bound
// on those, ncu r01).  2^128 = -2^32 (mod p), so top * C128 folds the third word back.
constexpr uint64_t C128 = 0xfffffffe00000001ull;   // 2^128 mod p

struct Wide { uint64_t lo, hi, top; };

__device__ __forceinline__ void wide_mac(Wide &A, uint64_t x, uint64_t y) {
    const uint64_t lo = x * y, hi = __umul64hi(x, y);
    asm("add.cc.u64 %0, %0, %3;\n\taddc.cc.u64 %1, %1, %4;\n\taddc.u64 %2, %2, 0;"
        : "+l"(A.lo), "+l"(A.hi), "+l"(A.top)
        : "l"(lo), "l"(hi));
}

__device__ __forceinline__ uint64_t wide_reduce(const Wide &A) {   // top < 2^32 (fewer than 2^32 products)
    return add(reduce128(A.hi, A.lo), mul(A.top, C128));
}

// x + y reduced only to 64 bits (congruent mod p, not necessarily canonical): a multiplication
// input needs no more.  Requires x < 2^64 and y < p (then x + y - 2^64 + 2^32 - 1 < 2^64); eval_pair
// only adds a canonical delta to a lazy value.
__device__ __forceinline__ uint64_t add_lazy(uint64_t x, uint64_t y) {
    const uint64_t s = x + y;
    return s < x ? s + EPS : s;       // x + y - 2^64 + (2^64 mod p) < 2^64
}

template <int D>
__device__ __forceinline__ void eval_pair(const uint64_t (&a)[D], const uint64_t (&b)[D], Wide (&acc)[D + 1]) {
    uint64_t v[D], dl[D];
#pragma unroll
    for (int m = 0; m < D; ++m) { v[m] = a[m]; dl[m] = sub(b[m], a[m]); }
#pragma unroll
    for (int t = 0; t <= D; ++t) {
        // v_m = a_m + t (b_m - a_m): t = 1 is b_m itself; later points are lazy sums (< 2^64)
        if (t == 1) {
#pragma unroll
            for (int m = 0; m < D; ++m) v[m] = b[m];
        } else if (t > 1) {
#pragma unroll
            for (int m = 0; m < D; ++m) v[m] = add_lazy(v[m], dl[m]);
        }
        if (D == 1) {
            wide_mac(acc[t], v[0], 1ull);
        } else {
            uint64_t prod = v[0];
#pragma unroll
            for (int m = 1; m + 1 < D; ++m) prod = mul(prod, v[m]);
            wide_mac(acc[t], prod, v[D - 1]);
        }
    }
}

__device__ __forceinline__ uint64_t fold(uint64_t a, uint64_t b, uint64_t r) { return add(a, mul(r, sub(b, a))); }

// transcript round over LE64 evaluations; r_i = LE64(state_i[0..8]) mod p  (reading R15)
template <int D>
__device__ __forceinline__ void finalize(uint64_t (&g)[D + 1], uint32_t round, State &ps, uint64_t *evals,
                                         uint64_t *chals, uint64_t *claim, bool given) {
    uint64_t r;
    if (given) {
        r = chals[round - 1];
    } else {
        sha256_words sh;
        sh.init();
#pragma unroll 1
        for (int i = 0; i < 8; ++i) sh.push(ps.st[i]);
#pragma unroll 1
        for (int t = 0; t <= D; ++t) { sh.push(bswap32((uint32_t)g[t])); sh.push(bswap32((uint32_t)(g[t] >> 32))); }
        uint32_t st[8];
        sh.finish(st);
#pragma unroll
        for (int i = 0; i < 8; ++i) ps.st[i] = st[i];
        r = (uint64_t)bswap32(st[0]) | ((uint64_t)bswap32(st[1]) << 32);
        if (r >= P) r -= P;
        chals[round - 1] = r;
    }
#pragma unroll
    for (int t = 0; t <= D; ++t) evals[(size_t)(round - 1) * (D + 1) + t] = g[t];
    if (round == 1 && claim) *claim = add(g[0], g[1]);
    ps.r = r;
}

struct Seed32Gl { uint8_t b[32]; };

static __global__ void k_gl_transcript_init(State *ps, uint32_t nproofs, Seed32Gl seed, const uint8_t *seeds,
                                            uint64_t first_index, uint32_t k, uint32_t d, uint32_t order) {
    uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= nproofs) return;
    uint32_t st[8];
    if (seeds) {
        Seed32Gl own;
        for (int i = 0; i < 32; ++i) own.b[i] = seeds[(size_t)b * 32 + i];
        transcript_init(st, own.b, first_index + b, k, d, order, 1u);
    } else {
        transcript_init(st, seed.b, first_index + b, k, d, order, 1u);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) ps[b].st[i] = st[i];
}

// ---------------------------------------------------------------- global round kernel

template <int D, int ORDER, bool FIRST>
__device__ __forceinline__ void load_pair(const uint64_t *src, uint64_t *dst, uint64_t h, uint64_t j, uint64_t r,
                                          uint64_t (&a)[D], uint64_t (&b)[D]) {
#pragma unroll
    for (int m = 0; m < D; ++m) {
        if (FIRST) {
            const uint64_t *T = src + (size_t)m * (2 * h);
            if (ORDER == 0) {
                const ulonglong2 v = __ldcs(reinterpret_cast<const ulonglong2 *>(T + 2 * j));
                a[m] = v.x; b[m] = v.y;
            } else {
                a[m] = __ldcs(T + j); b[m] = __ldcs(T + j + h);
            }
        } else {
            const uint64_t *T = src + (size_t)m * (4 * h);
            uint64_t *U = dst + (size_t)m * (2 * h);
            if (ORDER == 0) {
                const ulonglong2 v0 = __ldcs(reinterpret_cast<const ulonglong2 *>(T + 4 * j));
                const ulonglong2 v1 = __ldcs(reinterpret_cast<const ulonglong2 *>(T + 4 * j + 2));
                a[m] = fold(v0.x, v0.y, r);
                b[m] = fold(v1.x, v1.y, r);
                *reinterpret_cast<ulonglong2 *>(U + 2 * j) = make_ulonglong2(a[m], b[m]);
            } else {
                const uint64_t x0 = __ldcs(T + j), x1 = __ldcs(T + j + 2 * h);
                const uint64_t x2 = __ldcs(T + j + h), x3 = __ldcs(T + j + 3 * h);
                a[m] = fold(x0, x1, r);
                b[m] = fold(x2, x3, r);
                U[j] = a[m];
                U[j + h] = b[m];
            }
        }
    }
}

#ifndef GL_MLP
#define GL_MLP 4
#endif
#ifndef GL_OCC
#define GL_OCC 3
#endif
#ifndef GL_MLP_FUSED
#define GL_MLP_FUSED 2   // pairs per iteration of the split fused loop (g2: 2 -> fused 0.86 of HBM, 4 -> 0.83)
#endif

template <int D, int ORDER, bool FIRST>
__global__ void __launch_bounds__(256, GL_OCC) k_gl_round(RoundParams P) {
    __shared__ uint64_t s_red[32 * (D + 1)];
    __shared__ int s_last;
    const uint32_t b = blockIdx.y;
    const uint64_t h = 1ull << P.log_h;
    Wide wacc[D + 1];
#pragma unroll
    for (int t = 0; t <= D; ++t) wacc[t] = Wide{0, 0, 0};
#define GL_ACC wacc
    const uint64_t *src = P.src + (size_t)b * D * (FIRST ? 2 * h : 4 * h);
    uint64_t *dst = FIRST ? nullptr : P.dst + (size_t)b * D * (2 * h);
    const uint64_t r = FIRST ? 0 : P.ps[b].r;
    const uint64_t stride = (uint64_t)P.ctas * blockDim.x;
    uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // MLP pairs in flight per iteration (memory-level parallelism: the kernel streams); fewer for
    // d >= 3, whose wider accumulators would otherwise spill
    constexpr int MLP = D <= 2 ? GL_MLP : (GL_MLP > 2 ? 2 : GL_MLP);
    // fused rounds (both orders): all raw loads of the MLP pairs first (LSB fused rounds), then folds + stores, then evaluation:
    // every load is in flight before the first dependent instruction
    constexpr int MF = D <= 2 ? GL_MLP_FUSED : 2;
    if (!FIRST && ORDER == 0) {
        for (; j + (MF - 1) * stride < h; j += MF * stride) {
            ulonglong2 raw[MF][D][2];
#pragma unroll
            for (int q = 0; q < MF; ++q)
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    const uint64_t *T = src + (size_t)m * (4 * h) + 4 * (j + q * stride);
                    raw[q][m][0] = __ldcs(reinterpret_cast<const ulonglong2 *>(T));
                    raw[q][m][1] = __ldcs(reinterpret_cast<const ulonglong2 *>(T + 2));
                }
            uint64_t a[MF][D], bb[MF][D];
#pragma unroll
            for (int q = 0; q < MF; ++q)
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    a[q][m] = fold(raw[q][m][0].x, raw[q][m][0].y, r);
                    bb[q][m] = fold(raw[q][m][1].x, raw[q][m][1].y, r);
                    *reinterpret_cast<ulonglong2 *>(dst + (size_t)m * (2 * h) + 2 * (j + q * stride)) =
                        make_ulonglong2(a[q][m], bb[q][m]);
                }
#pragma unroll
            for (int q = 0; q < MF; ++q) eval_pair<D>(a[q], bb[q], GL_ACC);
        }
    }
    if (!FIRST && ORDER == 1) {
        // MSB (Alg. 1 pairing): fold pairs (x, x + 2h), this round pairs (j, j + h)
        for (; j + (MF - 1) * stride < h; j += MF * stride) {
            uint64_t x[MF][D][4];
#pragma unroll
            for (int q = 0; q < MF; ++q)
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    const uint64_t *T = src + (size_t)m * (4 * h) + (j + q * stride);
                    x[q][m][0] = __ldcs(T);
                    x[q][m][1] = __ldcs(T + 2 * h);
                    x[q][m][2] = __ldcs(T + h);
                    x[q][m][3] = __ldcs(T + 3 * h);
                }
            uint64_t a[MF][D], bb[MF][D];
#pragma unroll
            for (int q = 0; q < MF; ++q)
#pragma unroll
                for (int m = 0; m < D; ++m) {
                    a[q][m] = fold(x[q][m][0], x[q][m][1], r);
                    bb[q][m] = fold(x[q][m][2], x[q][m][3], r);
                    uint64_t *U = dst + (size_t)m * (2 * h);
                    U[j + q * stride] = a[q][m];
                    U[j + q * stride + h] = bb[q][m];
                }
#pragma unroll
            for (int q = 0; q < MF; ++q) eval_pair<D>(a[q], bb[q], GL_ACC);
        }
    }
    for (; j + (MLP - 1) * stride < h; j += MLP * stride) {
        uint64_t a[MLP][D], bb[MLP][D];
#pragma unroll
        for (int q = 0; q < MLP; ++q) load_pair<D, ORDER, FIRST>(src, dst, h, j + q * stride, r, a[q], bb[q]);
#pragma unroll
        for (int q = 0; q < MLP; ++q) eval_pair<D>(a[q], bb[q], GL_ACC);
    }
    for (; j < h; j += stride) {
        uint64_t a0[D], b0[D];
        load_pair<D, ORDER, FIRST>(src, dst, h, j, r, a0, b0);
        eval_pair<D>(a0, b0, GL_ACC);
    }
#undef GL_ACC
    uint64_t acc[D + 1];
#pragma unroll
    for (int t = 0; t <= D; ++t) acc[t] = wide_reduce(wacc[t]);
    block_reduce<D + 1>(acc, s_red);
    uint64_t *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    uint64_t *chals = P.challenges + (size_t)b * P.k;
    uint64_t *claim = P.claims ? P.claims + b : nullptr;
    if (P.ctas == 1) {
        if (threadIdx.x == 0) finalize<D>(acc, P.round, P.ps[b], evals, chals, claim, P.given);
        return;
    }
    uint64_t *part = P.partials + (size_t)b * P.ctas * (D + 1);
    if (threadIdx.x == 0) {
#pragma unroll
        for (int t = 0; t <= D; ++t) __stcg(&part[(size_t)blockIdx.x * (D + 1) + t], acc[t]);
        __threadfence();
        s_last = atomicAdd(&P.tickets[b], 1u) == P.ctas - 1;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int t = 0; t <= D; ++t) acc[t] = 0;
    for (uint32_t c = threadIdx.x; c < P.ctas; c += blockDim.x)
#pragma unroll
        for (int t = 0; t <= D; ++t) acc[t] = add(acc[t], __ldcg(&part[(size_t)c * (D + 1) + t]));
    block_reduce<D + 1>(acc, s_red);
    if (threadIdx.x == 0) {
        P.tickets[b] = 0;
        finalize<D>(acc, P.round, P.ps[b], evals, chals, claim, P.given);
    }
}

// ---------------------------------------------------------------- on-chip tail

template <int D, int ORDER>
__global__ void __launch_bounds__(256) k_gl_tail(TailParams P) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ uint64_t s_red[32 * (D + 1)];
    __shared__ uint64_t s_r;
    const uint32_t b = blockIdx.x;
    const uint32_t h0 = 1u << P.log_h0;
    uint64_t *A = reinterpret_cast<uint64_t *>(smem_raw);   // [D][2h0]
    uint64_t *Bf = A + (size_t)D * 2 * h0;                  // [D][h0]
    uint64_t *evals = P.round_evals + (size_t)b * P.k * (D + 1);
    uint64_t *chals = P.challenges + (size_t)b * P.k;
    uint64_t *claim = P.claims ? P.claims + b : nullptr;
    if (P.k == 0) {
        if (threadIdx.x == 0) {
            const uint64_t *src = P.src + (size_t)b * D;
            uint64_t prod = src[0];
            P.final_evals[(size_t)b * D] = prod;
            for (int m = 1; m < D; ++m) { P.final_evals[(size_t)b * D + m] = src[m]; prod = mul(prod, src[m]); }
            if (claim) *claim = prod;
        }
        return;
    }
    if (P.i0 == 1) {
        const uint64_t *src = P.src + (size_t)b * D * (2 * h0);
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) A[x] = src[x];
    } else {
        const uint64_t *src = P.src + (size_t)b * D * (4 * h0);
        const uint64_t r = P.ps[b].r;
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * 2 * h0; x += blockDim.x) {
            const uint32_t m = x / (2 * h0), y = x % (2 * h0);
            const uint64_t *T = src + (size_t)m * 4 * h0;
            A[x] = ORDER == 0 ? fold(T[2 * y], T[2 * y + 1], r) : fold(T[y], T[y + 2 * h0], r);
        }
    }
    __syncthreads();
    uint64_t *cur = A, *oth = Bf;
    uint32_t h = h0;
    for (uint32_t i = P.i0; i <= P.k; ++i) {
        uint64_t acc[D + 1];
#pragma unroll
        for (int t = 0; t <= D; ++t) acc[t] = 0;
        for (uint32_t j = threadIdx.x; j < h; j += blockDim.x) {
            uint64_t a[D], bb[D];
#pragma unroll
            for (int m = 0; m < D; ++m) {
                const uint64_t *T = cur + (size_t)m * 2 * h;
                a[m] = ORDER == 0 ? T[2 * j] : T[j];
                bb[m] = ORDER == 0 ? T[2 * j + 1] : T[j + h];
            }
            eval_pair<D>(a, bb, acc);
        }
        block_reduce<D + 1>(acc, s_red);
        if (threadIdx.x == 0) {
            finalize<D>(acc, i, P.ps[b], evals, chals, claim, P.given);
            s_r = P.ps[b].r;
        }
        __syncthreads();
        const uint64_t r = s_r;
        for (uint32_t x = threadIdx.x; x < (uint32_t)D * h; x += blockDim.x) {
            const uint32_t m = x / h, j = x % h;
            const uint64_t *T = cur + (size_t)m * 2 * h;
            oth[(size_t)m * h + j] = ORDER == 0 ? fold(T[2 * j], T[2 * j + 1], r) : fold(T[j], T[j + h], r);
        }
        __syncthreads();
        uint64_t *tmp = cur; cur = oth; oth = tmp;
        h >>= 1;
    }
    if (threadIdx.x < D) P.final_evals[(size_t)b * D + threadIdx.x] = cur[threadIdx.x];
}

}  // namespace gl

// launchers (k_gl.cu)
cudaError_t gl_launch_round(uint32_t D, uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                            const gl::RoundParams &p);
cudaError_t gl_launch_tail(uint32_t D, uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                           const gl::TailParams &p);
cudaError_t gl_launch_init(gl::State *ps, uint32_t nproofs, const uint8_t seed[32], const uint8_t *seeds_dev,
                           uint64_t first_index, uint32_t k, uint32_t d, uint32_t order, cudaStream_t s);
cudaError_t gl_set_attrs();

}  // namespace bzk
