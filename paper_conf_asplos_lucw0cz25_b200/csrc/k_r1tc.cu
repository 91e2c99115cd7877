// k_r1tc.cu -- instantiations of the tensor-core round kernels: d = 2 round 1 (round1_tc.cuh), d = 2
// fused rounds and d = 3 round 1 + fused rounds (fused_tc.cuh)
#include <stdlib.h>
#include "fused_tc.cuh"
#include "round1_tc.cuh"

namespace bzk {

// launch shape: NS stages of 16 KiB (one CTA per SM)
constexpr int kR1Stages = 12;

cudaError_t r1tc_launch(uint32_t order, bool sw64, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm) {
    if (order == 1) k_round1_tc<1, kR1Stages, false><<<grid, kR1Threads, r1_smem(kR1Stages), s>>>(p, tm);
    else if (sw64) k_round1_tc<0, kR1Stages, true><<<grid, kR1Threads, r1_smem(kR1Stages), s>>>(p, tm);
    else k_round1_tc<0, kR1Stages, false><<<grid, kR1Threads, r1_smem(kR1Stages), s>>>(p, tm);
    return cudaGetLastError();
}

template <int D, bool FIRST, int NW = ft_nw<D, FIRST>()>
static cudaError_t ftc_launch_t(uint32_t order, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm) {
    if (order == 1) k_fused_tc<D, 1, FIRST, NW><<<grid, ft_threads(NW), ft_smem<D, FIRST, NW>(), s>>>(p, tm);
    else k_fused_tc<D, 0, FIRST, NW><<<grid, ft_threads(NW), ft_smem<D, FIRST, NW>(), s>>>(p, tm);
    return cudaGetLastError();
}

cudaError_t ftc_launch(uint32_t D, bool first, bool small, uint32_t order, dim3 grid, cudaStream_t s,
                       const RoundParams &p, const CUtensorMap &tm) {
    if (D == 2 && !first) return small ? ftc_launch_t<2, false, kFtSmallNW>(order, grid, s, p, tm)
                                       : ftc_launch_t<2, false>(order, grid, s, p, tm);
    if (D == 3) return first ? ftc_launch_t<3, true>(order, grid, s, p, tm) : ftc_launch_t<3, false>(order, grid, s, p, tm);
    return cudaErrorInvalidValue;
}

template <int D, bool FIRST, int NW = ft_nw<D, FIRST>()>
static void ftc_attrs() {
    cudaFuncSetAttribute(k_fused_tc<D, 0, FIRST, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ft_smem<D, FIRST, NW>());
    cudaFuncSetAttribute(k_fused_tc<D, 1, FIRST, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ft_smem<D, FIRST, NW>());
}

cudaError_t r1tc_set_attrs() {
    ftc_attrs<2, false>();
    ftc_attrs<2, false, kFtSmallNW>();
    ftc_attrs<3, false>();
    ftc_attrs<3, true>();
    cudaFuncSetAttribute(k_round1_tc<0, kR1Stages, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)r1_smem(kR1Stages));
    cudaFuncSetAttribute(k_round1_tc<0, kR1Stages, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)r1_smem(kR1Stages));
    cudaFuncSetAttribute(k_round1_tc<1, kR1Stages, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)r1_smem(kR1Stages));
    return cudaGetLastError();
}

}  // namespace bzk
