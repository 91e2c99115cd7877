// k_enc.cu -- launchers of the encoder kernels (encoder.cuh).
#include "encoder.cuh"

namespace bzk {

cudaError_t enc_launch_spmv(dim3 grid, uint32_t threads, cudaStream_t s, const enc::SpmvParams &p) {
    enc::k_spmv<BZK_ENC_K, BZK_ENC_U><<<grid, threads, 0, s>>>(p);
    return cudaGetLastError();
}

cudaError_t enc_launch_to_mont(fe *v, uint64_t n, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    enc::k_to_mont<<<148 * 8, 256, 0, s>>>(v, n);
    return cudaGetLastError();
}

}  // namespace bzk
