// tc_probe_r1.cu -- standalone check of k_round1_tc's MMA: 6 tiles [a0][b0][D0][a1][b1][D1] of
// 128 rows x 32 bytes (32-byte swizzle), A = tiles 0..3 MN-major (M = 128), B = tiles 3..5 MN-major
// (N = 96), K = 128 rows in 4 instructions; D[128][96] vs the host product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -I paper_conf_asplos_lucw0cz25_b200/csrc \
//        scripts/tc_probe_r1.cu -o /tmp/tc_probe_r1 && /tmp/tc_probe_r1
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <vector>
#include "tc.cuh"

using namespace bzk;

__global__ void probe(const uint8_t *G, int32_t *D) {   // G: [6][128][32] plain
    extern __shared__ uint8_t raw[];
    uint8_t *base = raw + ((1024 - (tc::su32(raw) & 1023)) & 1023);
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t s_tmem;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp == 0) tc::tmem_alloc<256>(&s_tmem);
    if (threadIdx.x == 0) {
        tc::mbar_init_n(&bar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    for (int c = threadIdx.x; c < 6 * 128 * 2; c += blockDim.x) {
        const int t = c >> 8, j = (c >> 1) & 127, h = c & 1;
        uint8_t *dst = base + t * 4096 + j * 32 + ((h ^ ((j >> 2) & 1)) << 4);
        for (int i = 0; i < 16; ++i) dst[i] = G[(t * 128 + j) * 32 + h * 16 + i];
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = s_tmem;
    if (threadIdx.x == 0) {
        const uint32_t idesc = tc::idesc_u8(128, 96, true) | (1u << 15);
        const uint32_t a0 = tc::su32(base);
        for (int q = 0; q < 4; ++q)
            tc::mma_u8(tmem, tc::desc_sw32(a0 + q * 1024, 4096, 256), tc::desc_sw32(a0 + 12288 + q * 1024, 4096, 256),
                       idesc, q > 0);
        tc::commit(&bar);
    }
    __syncwarp();
    tc::mbar_wait(&bar, 0);
    tc::fence_after();
    uint32_t v[32];
    for (int c = 0; c < 3; ++c) {
        tc::ld_x32(tmem + ((uint32_t)(warp * 32) << 16) + c * 32, v);
        tc::wait_ld();
        for (int j = 0; j < 32; ++j) D[(warp * 32 + lane) * 96 + c * 32 + j] = (int32_t)v[j];
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc<256>(tmem);
}

int main() {
    std::vector<uint8_t> G(6 * 128 * 32);
    srand(3);
    for (auto &x : G) x = rand() & 255;
    uint8_t *Gd;
    int32_t *Dd;
    cudaMalloc(&Gd, G.size());
    cudaMalloc(&Dd, 128 * 96 * 4);
    cudaMemcpy(Gd, G.data(), G.size(), cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 32 * 1024);
    probe<<<1, 128, 32 * 1024>>>(Gd, Dd);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("kernel error %s\n", cudaGetErrorString(e)); return 1; }
    std::vector<int32_t> D(128 * 96);
    cudaMemcpy(D.data(), Dd, D.size() * 4, cudaMemcpyDeviceToHost);
    long bad = 0;
    for (int r = 0; r < 128; ++r)
        for (int c = 0; c < 96; ++c) {
            long s = 0;
            for (int j = 0; j < 128; ++j) s += (long)G[((r / 32) * 128 + j) * 32 + r % 32] * G[((3 + c / 32) * 128 + j) * 32 + c % 32];
            if (s != D[r * 96 + c] && bad++ < 8) printf("D[%d][%d] = %d want %ld\n", r, c, D[r * 96 + c], s);
        }
    printf("r1 mismatches %ld / %d\n", bad, 128 * 96);
    return bad ? 2 : 0;
}
