// k_r1tc.cu -- instantiations of the tensor-core round-1 kernel for d = 2 (round1_tc.cuh)
#include "round1_tc.cuh"

namespace bzk {

cudaError_t r1tc_launch(uint32_t order, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm) {
    if (order == 1) k_round1_tc<1><<<grid, kR1Threads, kR1Smem, s>>>(p, tm);
    else k_round1_tc<0><<<grid, kR1Threads, kR1Smem, s>>>(p, tm);
    return cudaGetLastError();
}

cudaError_t r1tc_set_attrs() {
    cudaFuncSetAttribute(k_round1_tc<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kR1Smem);
    return cudaFuncSetAttribute(k_round1_tc<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kR1Smem);
}

}  // namespace bzk
