// k_multi.cu -- instantiations of the known-challenge multi-round pass (multiround.cuh, NEXT-1)
#include "multiround.cuh"
#include <stdlib.h>
#include "multiround_tc.cuh"

namespace bzk {

template <int M>
constexpr size_t multi_tma_smem() { return (size_t)8 * (1u << M) * 1024 + 1024; }   // 8 warps x 2^M KiB + align

template <int ORDER, bool TMA>
static cudaError_t multi_launch_o(uint32_t m, dim3 grid, cudaStream_t s, const MultiParams &p, const CUtensorMap &tm) {
    switch (m) {
        case 1: k_multi<ORDER, 1, TMA><<<grid, 256, TMA ? multi_tma_smem<1>() : 0, s>>>(p, tm); break;
        case 2: k_multi<ORDER, 2, TMA><<<grid, 256, TMA ? multi_tma_smem<2>() : 0, s>>>(p, tm); break;
        case 3: k_multi<ORDER, 3, TMA><<<grid, 256, TMA ? multi_tma_smem<3>() : 0, s>>>(p, tm); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t multi_launch(uint32_t order, uint32_t m, bool tma, dim3 grid, cudaStream_t s, const MultiParams &p,
                         const CUtensorMap &tm) {
    if (order == 0) return multi_launch_o<0, false>(m, grid, s, p, tm);
    return tma ? multi_launch_o<1, true>(m, grid, s, p, tm) : multi_launch_o<1, false>(m, grid, s, p, tm);
}

// k_multi_tc launch shape (NS stages, EG epilogue groups, CM rows of the column-sum product).  Sweep
// on B200 (m0lit, profiles/r02/bench_m0lit_cfg*_r02tcs.json): (4,2,128) (4,2,64) (6,2,64) (4,4,64)
// (6,4,64) (6,3,64) all 8.9-9.0 ms per step -- the passes stream at the TMA/HBM rate whatever the
// pipeline depth or epilogue width; the simplest shape is kept.
#define BZK_TC_SHAPES(X) X(4, 2, 128)
static int tc_cfg() { return 0; }

cudaError_t multi_tc_launch(uint32_t order, dim3 grid, cudaStream_t s, const MultiParams &p, const CUtensorMap &tm) {
    int i = 0;
#define BZK_TC_LAUNCH(NS, EG, CM)                                                                        \
    if (tc_cfg() == i++) {                                                                              \
        if (order == 1) k_multi_tc<1, NS, EG, CM><<<grid, tc_threads(EG), tc_smem(NS), s>>>(p, tm);       \
        else k_multi_tc<0, NS, EG, CM><<<grid, tc_threads(EG), tc_smem(NS), s>>>(p, tm);                   \
        return cudaGetLastError();                                                                      \
    }
    BZK_TC_SHAPES(BZK_TC_LAUNCH)
#undef BZK_TC_LAUNCH
    return cudaErrorInvalidValue;
}

cudaError_t multi_set_attrs() {
#define BZK_TC_ATTR(NS, EG, CM)                                                                                   \
    cudaFuncSetAttribute(k_multi_tc<0, NS, EG, CM>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tc_smem(NS)); \
    cudaFuncSetAttribute(k_multi_tc<1, NS, EG, CM>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tc_smem(NS));
    BZK_TC_SHAPES(BZK_TC_ATTR)
#undef BZK_TC_ATTR
    cudaFuncSetAttribute(k_multi<1, 1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)multi_tma_smem<1>());
    cudaFuncSetAttribute(k_multi<1, 2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)multi_tma_smem<2>());
    return cudaFuncSetAttribute(k_multi<1, 3, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)multi_tma_smem<3>());
}

}  // namespace bzk
