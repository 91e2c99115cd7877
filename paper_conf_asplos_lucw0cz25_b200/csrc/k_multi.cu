// k_multi.cu -- instantiations of the known-challenge multi-round pass (multiround.cuh, NEXT-1)
#include "multiround.cuh"

namespace bzk {

template <int ORDER>
static cudaError_t multi_launch_o(uint32_t m, dim3 grid, cudaStream_t s, const MultiParams &p) {
    switch (m) {
        case 1: k_multi<ORDER, 1><<<grid, 256, 0, s>>>(p); break;
        case 2: k_multi<ORDER, 2><<<grid, 256, 0, s>>>(p); break;
        case 3: k_multi<ORDER, 3><<<grid, 256, 0, s>>>(p); break;
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t multi_launch(uint32_t order, uint32_t m, dim3 grid, cudaStream_t s, const MultiParams &p) {
    return order == 0 ? multi_launch_o<0>(m, grid, s, p) : multi_launch_o<1>(m, grid, s, p);
}

}  // namespace bzk
