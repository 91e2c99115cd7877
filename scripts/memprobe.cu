// memprobe.cu -- DRAM-traffic probe for the fused-round access pattern (run under ncu, one GPU).
// Each variant streams the same 4 GiB source; ncu's dram__bytes_read/write per launch shows which
// access pattern costs extra DRAM reads.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 memprobe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

struct e32 { uint32_t w[8]; };
__device__ __forceinline__ e32 ld8(const e32 *p) {
    e32 r;
    asm volatile("ld.global.cs.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];" : "=r"(r.w[0]), "=r"(r.w[1]), "=r"(r.w[2]),
                 "=r"(r.w[3]), "=r"(r.w[4]), "=r"(r.w[5]), "=r"(r.w[6]), "=r"(r.w[7]) : "l"(p));
    return r;
}
__device__ __forceinline__ void st8(e32 *p, const e32 &v) {
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v.w[0]), "r"(v.w[1]), "r"(v.w[2]),
                 "r"(v.w[3]), "r"(v.w[4]), "r"(v.w[5]), "r"(v.w[6]), "r"(v.w[7]) : "memory");
}
__device__ __forceinline__ e32 mix(const e32 &a, const e32 &b) {
    e32 r;
    for (int i = 0; i < 8; ++i) r.w[i] = a.w[i] ^ (b.w[i] * 3u);
    return r;
}

// V: 0 = 4 consecutive per thread, read only;  1 = 2 consecutive per thread, read only
//    2 = 4 consecutive per thread + 2 consecutive written;  3 = coalesced lanes (lane + 32q) read + write
//    4 = 4 consecutive read + 2 written with st.global.cs
template <int V>
__global__ void __launch_bounds__(256) k(const e32 *src, e32 *dst, uint64_t n_groups, uint32_t *sink) {
    uint32_t acc = 0;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n_groups; j += stride) {
        if (V == 1) {
            e32 a = ld8(src + 2 * j), b = ld8(src + 2 * j + 1);
            acc ^= mix(a, b).w[0];
        } else if (V == 3) {
            const uint64_t w = j / 32, l = j % 32;   // warp w covers 128 consecutive elements
            e32 x[4];
            for (int q = 0; q < 4; ++q) x[q] = ld8(src + 128 * w + l + 32 * q);
            st8(dst + 64 * w + l, mix(x[0], x[1]));
            st8(dst + 64 * w + l + 32, mix(x[2], x[3]));
        } else {
            e32 x0 = ld8(src + 4 * j), x1 = ld8(src + 4 * j + 1), x2 = ld8(src + 4 * j + 2), x3 = ld8(src + 4 * j + 3);
            if (V == 0) acc ^= mix(mix(x0, x1), mix(x2, x3)).w[0];
            else if (V == 2) { st8(dst + 2 * j, mix(x0, x1)); st8(dst + 2 * j + 1, mix(x2, x3)); }
            else {
                e32 lo = mix(x0, x1), hi = mix(x2, x3);
                asm volatile("st.global.cs.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst + 2 * j), "r"(lo.w[0]), "r"(lo.w[1]), "r"(lo.w[2]), "r"(lo.w[3]), "r"(lo.w[4]), "r"(lo.w[5]), "r"(lo.w[6]), "r"(lo.w[7]) : "memory");
                asm volatile("st.global.cs.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(dst + 2 * j + 1), "r"(hi.w[0]), "r"(hi.w[1]), "r"(hi.w[2]), "r"(hi.w[3]), "r"(hi.w[4]), "r"(hi.w[5]), "r"(hi.w[6]), "r"(hi.w[7]) : "memory");
            }
        }
    }
    if (acc == 0x12345678u) sink[0] = acc;
}

int main() {
    const uint64_t bytes = 4ull << 30, n = bytes / 32;
    e32 *src, *dst;
    uint32_t *sink;
    cudaMalloc(&src, bytes);
    cudaMalloc(&dst, bytes / 2);
    cudaMalloc(&sink, 4);
    cudaMemset(src, 1, bytes);
    cudaMemset(dst, 0, bytes / 2);
    const int grid = 148 * 2 * 4;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int rep = 0; rep < 2; ++rep) {
        float ms[5];
        cudaEventRecord(e0); k<0><<<grid, 256>>>(src, dst, n / 4, sink); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms[0], e0, e1);
        cudaEventRecord(e0); k<1><<<grid, 256>>>(src, dst, n / 2, sink); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms[1], e0, e1);
        cudaEventRecord(e0); k<2><<<grid, 256>>>(src, dst, n / 4, sink); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms[2], e0, e1);
        cudaEventRecord(e0); k<3><<<grid, 256>>>(src, dst, n / 4, sink); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms[3], e0, e1);
        cudaEventRecord(e0); k<4><<<grid, 256>>>(src, dst, n / 4, sink); cudaEventRecord(e1); cudaEventSynchronize(e1); cudaEventElapsedTime(&ms[4], e0, e1);
        for (int v = 0; v < 5; ++v) {
            const double moved = (v == 0 || v == 1) ? bytes : 1.5 * bytes;
            printf("variant %d: %.3f ms  %.0f GB/s (algorithmic)\n", v, ms[v], moved / (ms[v] * 1e-3) / 1e9);
        }
    }
    printf("err: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
