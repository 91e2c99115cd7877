// k_impl.cuh -- per-degree kernel instantiation; included by k_d1.cu .. k_d4.cu with BZK_D set.
#include "sumcheck.cuh"
#include "small.cuh"

namespace bzk {

template <int ORDER, bool FIRST, bool TMA>
static cudaError_t launch_round_v(dim3 grid, uint32_t threads, cudaStream_t s, const RoundParams &p,
                                  const CUtensorMap &tm) {
    const size_t sm = TMA ? tma_smem_bytes<BZK_D, FIRST>() : 0;
    if (p.cluster <= 1) {
        k_round<BZK_D, ORDER, FIRST, TMA><<<grid, threads, sm, s>>>(p, tm);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(threads, 1, 1);
    cfg.dynamicSmemBytes = sm;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = p.cluster;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_round<BZK_D, ORDER, FIRST, TMA>, p, tm);
}

template <bool TMA>
static cudaError_t launch_round_t(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                                  const RoundParams &p, const CUtensorMap &tm) {
    if (order == 0) return first ? launch_round_v<0, true, TMA>(grid, threads, s, p, tm)
                                 : launch_round_v<0, false, TMA>(grid, threads, s, p, tm);
    return first ? launch_round_v<1, true, TMA>(grid, threads, s, p, tm)
                 : launch_round_v<1, false, TMA>(grid, threads, s, p, tm);
}

template <>
cudaError_t launch_round<BZK_D>(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                                const RoundParams &p, const CUtensorMap &tm) {
    return p.tma ? launch_round_t<true>(order, first, grid, threads, s, p, tm)
                 : launch_round_t<false>(order, first, grid, threads, s, p, tm);
}

template <int ORDER, bool FIRST>
static void set_round_attrs() {
    cudaFuncSetAttribute(k_round<BZK_D, ORDER, FIRST, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)tma_smem_bytes<BZK_D, FIRST>());
}

template <>
cudaError_t set_kernel_attrs<BZK_D>() {
    set_round_attrs<0, true>();
    set_round_attrs<0, false>();
    set_round_attrs<1, true>();
    set_round_attrs<1, false>();
    cudaFuncSetAttribute(k_small<BZK_D, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_small<BZK_D, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_tail<BZK_D, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    return cudaFuncSetAttribute(k_tail<BZK_D, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

template <>
cudaError_t launch_small<BZK_D>(uint32_t order, dim3 grid, uint32_t cs, size_t smem, cudaStream_t s,
                                const SmallParams &p) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(256, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return order == 0 ? cudaLaunchKernelEx(&cfg, k_small<BZK_D, 0>, p) : cudaLaunchKernelEx(&cfg, k_small<BZK_D, 1>, p);
}

template <>
cudaError_t launch_tail<BZK_D>(uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                               const TailParams &p) {
    if (order == 0) k_tail<BZK_D, 0><<<grid, threads, smem, s>>>(p);
    else            k_tail<BZK_D, 1><<<grid, threads, smem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace bzk
