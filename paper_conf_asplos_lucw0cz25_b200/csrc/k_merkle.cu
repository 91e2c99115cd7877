// k_merkle.cu -- launchers of the Merkle stage kernel (merkle.cuh), every hash mode and
// per-thread subtree height (0..4) in one translation unit.
#include "merkle.cuh"

namespace bzk {

template <int MODE>
static cudaError_t stage_mode(uint32_t lt, uint32_t grid, uint32_t threads, cudaStream_t s,
                              const mk::StageParams &p) {
    switch (lt) {
        case 0: mk::k_merkle_stage<MODE, 0><<<grid, threads, 0, s>>>(p); break;
        case 1: mk::k_merkle_stage<MODE, 1><<<grid, threads, 0, s>>>(p); break;
        case 2: mk::k_merkle_stage<MODE, 2><<<grid, threads, 0, s>>>(p); break;
        case 3: mk::k_merkle_stage<MODE, 3><<<grid, threads, 0, s>>>(p); break;
        case 4: mk::k_merkle_stage<MODE, 4><<<grid, threads, 0, s>>>(p); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t merkle_launch_stage(uint32_t mode, uint32_t lt, uint32_t grid, uint32_t threads, cudaStream_t s,
                                const mk::StageParams &p) {
    return mode == 1 ? stage_mode<1>(lt, grid, threads, s, p) : stage_mode<0>(lt, grid, threads, s, p);
}

}  // namespace bzk
