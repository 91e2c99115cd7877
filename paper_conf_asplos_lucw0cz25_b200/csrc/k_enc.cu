// k_enc.cu -- launchers of the encoder kernels (encoder.cuh).
#include "encoder.cuh"

namespace bzk {

cudaError_t enc_launch_spmv(dim3 grid, uint32_t threads, cudaStream_t s, const enc::SpmvParams &p) {
#if BZK_ENC_ASYNC
    const size_t smem = (size_t)BZK_ENC_S * (BZK_ENC_K + 1) * 2 * 16 * threads;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(enc::k_spmv_async<BZK_ENC_K, BZK_ENC_S>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem);
        attr = true;
    }
    enc::k_spmv_async<BZK_ENC_K, BZK_ENC_S><<<grid, threads, smem, s>>>(p);
#else
    enc::k_spmv<BZK_ENC_K, BZK_ENC_U><<<grid, threads, 0, s>>>(p);
#endif
    return cudaGetLastError();
}

cudaError_t enc_launch_to_mont(fe *v, uint64_t n, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    enc::k_to_mont<<<148 * 8, 256, 0, s>>>(v, n);
    return cudaGetLastError();
}

}  // namespace bzk
