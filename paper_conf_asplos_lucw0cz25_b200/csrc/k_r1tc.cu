// k_r1tc.cu -- instantiations of the tensor-core round kernels: d = 2 round 1 (round1_tc.cuh), d = 2
// fused rounds and d = 3 round 1 + fused rounds (fused_tc.cuh)
#include <stdlib.h>
#include "fused_tc.cuh"
#include "round1_tc.cuh"

namespace bzk {

// launch shape: 6 stages, 4 D-prep warps.  Sweep on B200 (c2 round 1 per step, profiles/r02/
// bench_c2_r1cfg*_r02r1s.json): (6, 2) 14.6 ms, (8, 2) 15.2, (6, 4) 11.6, (8, 4) 11.7 -- the D = b + p - a
// pass sits on every stage's critical path, so its width matters and the stage count does not.
#define BZK_R1_SHAPES(X) X(6, 4)
static int r1_cfg() { return 0; }

cudaError_t r1tc_launch(uint32_t order, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm) {
    int i = 0;
#define BZK_R1_LAUNCH(NS, PW)                                                                            \
    if (r1_cfg() == i++) {                                                                              \
        if (order == 1) k_round1_tc<1, NS, PW><<<grid, r1_threads(PW), r1_smem(NS), s>>>(p, tm);          \
        else k_round1_tc<0, NS, PW><<<grid, r1_threads(PW), r1_smem(NS), s>>>(p, tm);                      \
        return cudaGetLastError();                                                                      \
    }
    BZK_R1_SHAPES(BZK_R1_LAUNCH)
#undef BZK_R1_LAUNCH
    return cudaErrorInvalidValue;
}

template <int D, bool FIRST>
static cudaError_t ftc_launch_t(uint32_t order, dim3 grid, cudaStream_t s, const RoundParams &p, const CUtensorMap &tm) {
    if (order == 1) k_fused_tc<D, 1, FIRST><<<grid, ft_threads<D, FIRST>(), ft_smem<D, FIRST>(), s>>>(p, tm);
    else k_fused_tc<D, 0, FIRST><<<grid, ft_threads<D, FIRST>(), ft_smem<D, FIRST>(), s>>>(p, tm);
    return cudaGetLastError();
}

cudaError_t ftc_launch(uint32_t D, bool first, uint32_t order, dim3 grid, cudaStream_t s, const RoundParams &p,
                       const CUtensorMap &tm) {
    if (D == 2 && !first) return ftc_launch_t<2, false>(order, grid, s, p, tm);
    if (D == 3) return first ? ftc_launch_t<3, true>(order, grid, s, p, tm) : ftc_launch_t<3, false>(order, grid, s, p, tm);
    return cudaErrorInvalidValue;
}

template <int D, bool FIRST>
static void ftc_attrs() {
    cudaFuncSetAttribute(k_fused_tc<D, 0, FIRST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ft_smem<D, FIRST>());
    cudaFuncSetAttribute(k_fused_tc<D, 1, FIRST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ft_smem<D, FIRST>());
}

cudaError_t r1tc_set_attrs() {
    ftc_attrs<2, false>();
    ftc_attrs<3, false>();
    ftc_attrs<3, true>();
#define BZK_R1_ATTR(NS, PW)                                                                                  \
    cudaFuncSetAttribute(k_round1_tc<0, NS, PW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)r1_smem(NS)); \
    cudaFuncSetAttribute(k_round1_tc<1, NS, PW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)r1_smem(NS));
    BZK_R1_SHAPES(BZK_R1_ATTR)
#undef BZK_R1_ATTR
    return cudaGetLastError();
}

}  // namespace bzk
