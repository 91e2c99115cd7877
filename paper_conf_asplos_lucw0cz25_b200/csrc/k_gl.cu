// k_gl.cu -- launchers of the Goldilocks kernels (gl.cuh), all degrees and orders in one unit.
#include <string.h>
#include "gl.cuh"

namespace bzk {

template <int D>
static cudaError_t round_d(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                           const gl::RoundParams &p) {
    if (order == 0) {
        if (first) gl::k_gl_round<D, 0, true><<<grid, threads, 0, s>>>(p);
        else       gl::k_gl_round<D, 0, false><<<grid, threads, 0, s>>>(p);
    } else {
        if (first) gl::k_gl_round<D, 1, true><<<grid, threads, 0, s>>>(p);
        else       gl::k_gl_round<D, 1, false><<<grid, threads, 0, s>>>(p);
    }
    return cudaGetLastError();
}

template <int D>
static cudaError_t tail_d(uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                          const gl::TailParams &p) {
    if (order == 0) gl::k_gl_tail<D, 0><<<grid, threads, smem, s>>>(p);
    else            gl::k_gl_tail<D, 1><<<grid, threads, smem, s>>>(p);
    return cudaGetLastError();
}

cudaError_t gl_launch_round(uint32_t D, uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                            const gl::RoundParams &p) {
    switch (D) {
        case 1: return round_d<1>(order, first, grid, threads, s, p);
        case 2: return round_d<2>(order, first, grid, threads, s, p);
        case 3: return round_d<3>(order, first, grid, threads, s, p);
        case 4: return round_d<4>(order, first, grid, threads, s, p);
    }
    return cudaErrorInvalidValue;
}

cudaError_t gl_launch_tail(uint32_t D, uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                           const gl::TailParams &p) {
    switch (D) {
        case 1: return tail_d<1>(order, grid, threads, smem, s, p);
        case 2: return tail_d<2>(order, grid, threads, smem, s, p);
        case 3: return tail_d<3>(order, grid, threads, smem, s, p);
        case 4: return tail_d<4>(order, grid, threads, smem, s, p);
    }
    return cudaErrorInvalidValue;
}

cudaError_t gl_launch_init(gl::State *ps, uint32_t nproofs, const uint8_t seed[32], const uint8_t *seeds_dev,
                           uint64_t first_index, uint32_t k, uint32_t d, uint32_t order, cudaStream_t s) {
    gl::Seed32Gl sd;
    memset(sd.b, 0, 32);
    if (seed) memcpy(sd.b, seed, 32);
    gl::k_gl_transcript_init<<<(nproofs + 127) / 128, 128, 0, s>>>(ps, nproofs, sd, seeds_dev, first_index, k, d, order);
    return cudaGetLastError();
}

template <int D>
static void attrs_d() {
    cudaFuncSetAttribute(gl::k_gl_tail<D, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(gl::k_gl_tail<D, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

cudaError_t gl_set_attrs() {
    attrs_d<1>(); attrs_d<2>(); attrs_d<3>(); attrs_d<4>();
    return cudaGetLastError();
}

}  // namespace bzk
