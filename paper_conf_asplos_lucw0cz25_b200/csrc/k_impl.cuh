// k_impl.cuh -- per-degree kernel instantiation; included by k_d1.cu .. k_d4.cu with BZK_D set.
#include "sumcheck.cuh"

namespace bzk {

template <int ORDER, bool FIRST>
static cudaError_t launch_round_cl(dim3 grid, uint32_t threads, size_t sm, cudaStream_t s, const RoundParams &p,
                                   uint32_t cluster) {
    if (cluster <= 1) {
        k_round<BZK_D, ORDER, FIRST><<<grid, threads, sm, s>>>(p);
        return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(threads, 1, 1);
    cfg.dynamicSmemBytes = sm;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = cluster;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_round<BZK_D, ORDER, FIRST>, p);
}

template <>
cudaError_t launch_round<BZK_D>(uint32_t order, bool first, dim3 grid, uint32_t threads, cudaStream_t s,
                                const RoundParams &p) {
    const size_t sm = 0;
    const uint32_t cl = p.cluster;
    if (order == 0) return first ? launch_round_cl<0, true>(grid, threads, sm, s, p, cl)
                                 : launch_round_cl<0, false>(grid, threads, sm, s, p, cl);
    return first ? launch_round_cl<1, true>(grid, threads, sm, s, p, cl)
                 : launch_round_cl<1, false>(grid, threads, sm, s, p, cl);
}

template <>
cudaError_t set_kernel_attrs<BZK_D>() {
    const int big = 200 * 1024;
    cudaFuncSetAttribute(k_round<BZK_D, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
    cudaFuncSetAttribute(k_round<BZK_D, 1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
    cudaFuncSetAttribute(k_round<BZK_D, 0, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
    cudaFuncSetAttribute(k_round<BZK_D, 1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
    cudaFuncSetAttribute(k_tail<BZK_D, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    return cudaFuncSetAttribute(k_tail<BZK_D, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

template <>
cudaError_t launch_tail<BZK_D>(uint32_t order, uint32_t grid, uint32_t threads, size_t smem, cudaStream_t s,
                               const TailParams &p) {
    if (order == 0) k_tail<BZK_D, 0><<<grid, threads, smem, s>>>(p);
    else            k_tail<BZK_D, 1><<<grid, threads, smem, s>>>(p);
    return cudaGetLastError();
}

}  // namespace bzk
