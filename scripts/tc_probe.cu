// tc_probe.cu -- standalone check of the tcgen05 kind::i8 layouts k_multi_tc relies on (one CTA, one
// 128-row tile): a 3-D TMA box with 32-byte rows and the 32-byte swizzle lands as a K-major A operand
// (8 segments of 128 x 32 bytes), a hand-swizzled K-major B operand (8 x 64 x 32 bytes), and the same
// tile read again as an MN-major B operand against an all-ones A for the column byte sums.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -I paper_conf_asplos_lucw0cz25_b200/csrc \
//        scripts/tc_probe.cu -o /tmp/tc_probe && /tmp/tc_probe
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <vector>
#include "tc.cuh"

using namespace bzk;

__global__ void probe(const __grid_constant__ CUtensorMap tm, const uint8_t *Bg, int32_t *D, int32_t *D2) {
    extern __shared__ uint8_t raw[];
    uint8_t *base = raw + ((1024 - (tc::su32(raw) & 1023)) & 1023);
    uint8_t *A = base;                 // 8 x 4 KiB
    uint8_t *B = base + 32768;         // 8 x 2 KiB
    uint8_t *ones = base + 49152;      // 4 KiB
    __shared__ __align__(8) uint64_t bar_tma, bar_mma;
    __shared__ uint32_t s_tmem;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) tc::tmem_alloc<512>(&s_tmem);
    if (threadIdx.x == 0) {
        tc::mbar_init_n(&bar_tma, 1);
        tc::mbar_init_n(&bar_mma, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int c = threadIdx.x; c < 8 * 64 * 2; c += blockDim.x) {   // 16-byte chunks of B, 32B swizzle
        const int z = c >> 7, n = (c >> 1) & 63, h = c & 1;
        uint8_t *dst = B + z * 2048 + n * 32 + ((h ^ ((n >> 2) & 1)) << 4);
        for (int i = 0; i < 16; ++i) dst[i] = Bg[(z * 64 + n) * 32 + h * 16 + i];
    }
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) ones[i] = 1;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    if (threadIdx.x == 0) {
        tc::mbar_tx(&bar_tma, 32768);
        tc::tma3(A, &tm, 0, 0, 0, &bar_tma);
        tc::mbar_wait(&bar_tma, 0);
        tc::fence_after();
        const uint32_t id_main = tc::idesc_u8(128, 64, false), id_col = tc::idesc_u8(128, 256, true);
        for (int z = 0; z < 8; ++z)
            tc::mma_u8(tmem, tc::desc_sw32(tc::su32(A + z * 4096), 16, 256), tc::desc_sw32(tc::su32(B + z * 2048), 16, 256),
                       id_main, z > 0);
        for (int q = 0; q < 4; ++q)
            tc::mma_u8(tmem + 256, tc::desc_sw32(tc::su32(ones), 16, 256), tc::desc_sw32(tc::su32(A + q * 1024), 4096, 256),
                       id_col, q > 0);
        tc::commit(&bar_mma);
    }
    __syncwarp();
    tc::mbar_wait(&bar_mma, 0);
    tc::fence_after();
    const int row = warp * 32 + lane;
    const uint32_t ta = tmem + ((uint32_t)(warp * 32) << 16);
    uint32_t v[32];
    for (int c = 0; c < 2; ++c) {
        tc::ld_x32(ta + c * 32, v);
        tc::wait_ld();
        for (int j = 0; j < 32; ++j) D[row * 64 + c * 32 + j] = (int32_t)v[j];
    }
    for (int c = 0; c < 8; ++c) {
        tc::ld_x32(ta + 256 + c * 32, v);
        tc::wait_ld();
        for (int j = 0; j < 32; ++j) D2[row * 256 + c * 32 + j] = (int32_t)v[j];
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<512>(tmem);
}

int main() {
    const int Ny = 128, Z = 8;
    std::vector<uint8_t> Ah(Z * Ny * 32), Bh(Z * 64 * 32);
    srand(7);
    for (auto &x : Ah) x = rand() & 255;
    for (auto &x : Bh) x = rand() & 255;
    for (int i = 0; i < 32; ++i) Ah[i] = 255, Bh[i] = 255;   // extremes
    uint8_t *Ad, *Bd;
    int32_t *Dd, *D2d;
    cudaMalloc(&Ad, Ah.size());
    cudaMalloc(&Bd, Bh.size());
    cudaMalloc(&Dd, 128 * 64 * 4);
    cudaMalloc(&D2d, 128 * 256 * 4);
    cudaMemcpy(Ad, Ah.data(), Ah.size(), cudaMemcpyHostToDevice);
    cudaMemcpy(Bd, Bh.data(), Bh.size(), cudaMemcpyHostToDevice);
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    CUtensorMap tm;
    cuuint64_t dims[3] = {8, (cuuint64_t)Ny, (cuuint64_t)Z};
    cuuint64_t strides[2] = {32, (cuuint64_t)Ny * 32};
    cuuint32_t box[3] = {8, 128, 8}, es[3] = {1, 1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 3, Ad, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); return 1; }
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 60 * 1024);
    probe<<<1, 128, 60 * 1024>>>(tm, Bd, Dd, D2d);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("kernel error %s\n", cudaGetErrorString(e)); return 1; }
    std::vector<int32_t> D(128 * 64), D2(128 * 256);
    cudaMemcpy(D.data(), Dd, D.size() * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(D2.data(), D2d, D2.size() * 4, cudaMemcpyDeviceToHost);
    long bad = 0, bad2 = 0;
    for (int y = 0; y < 128; ++y)
        for (int n = 0; n < 64; ++n) {
            long s = 0;
            for (int z = 0; z < Z; ++z)
                for (int i = 0; i < 32; ++i) s += (long)Ah[(z * Ny + y) * 32 + i] * Bh[(z * 64 + n) * 32 + i];
            if (s != D[y * 64 + n] && bad++ < 5) printf("D[%d][%d] = %d want %ld\n", y, n, D[y * 64 + n], s);
        }
    for (int z = 0; z < Z; ++z)
        for (int i = 0; i < 32; ++i) {
            long s = 0;
            for (int y = 0; y < Ny; ++y) s += Ah[(z * Ny + y) * 32 + i];
            for (int m = 0; m < 128; ++m)
                if (s != D2[m * 256 + z * 32 + i] && bad2++ < 5)
                    printf("D2[%d][%d] = %d want %ld\n", m, z * 32 + i, D2[m * 256 + z * 32 + i], s);
        }
    printf("main mismatches %ld / %d, colsum mismatches %ld / %d\n", bad, 128 * 64, bad2, 128 * 256);
    return (bad || bad2) ? 2 : 0;
}
