// gen.cuh -- device twin of paper_conf_asplos_lucw0cz25_b200/inputs.py (counter-based SplitMix64).
// Holds no field arithmetic: it turns (I, m, x, w) into 64-bit words exactly as inputs.py does.
#pragma once
#include <stdint.h>

namespace bzk {

__device__ __forceinline__ uint64_t splitmix64_ctr(uint64_t ctr, uint64_t seed) {
    uint64_t z = seed + (ctr + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// dst: [batch][d][2^k][4] u64; one thread per element (4 words, stored as 2 x 16 B)
static __global__ void k_generate(uint64_t *dst, uint64_t batch, uint32_t d, uint32_t k, uint64_t first_index,
                           uint32_t dist, uint64_t seed) {
    const uint64_t N = 1ull << k;
    const uint64_t total = batch * d * N;
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
         e += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t x = e & (N - 1);
        uint64_t bm = e >> k;
        uint64_t m = bm % d, b = bm / d;
        uint64_t I = first_index + b;
        uint64_t base = (I << 36) | (m << 32) | (x << 2);
        if (dist == 3) {   // Goldilocks: one word per element, masked to 63 bits
            dst[e] = splitmix64_ctr(base, seed) & ((1ull << 63) - 1);
            continue;
        }
        bool small = dist == 1 || (dist == 2 && m == 0);
        uint64_t w0, w1, w2, w3;
        if (small) {
            w0 = splitmix64_ctr(base, seed) & 0xffull;
            w1 = w2 = w3 = 0;
        } else {
            w0 = splitmix64_ctr(base | 0, seed);
            w1 = splitmix64_ctr(base | 1, seed);
            w2 = splitmix64_ctr(base | 2, seed);
            w3 = splitmix64_ctr(base | 3, seed) & ((1ull << 61) - 1);
        }
        ulonglong2 *q = reinterpret_cast<ulonglong2 *>(dst + 4 * e);
        q[0] = make_ulonglong2(w0, w1);
        q[1] = make_ulonglong2(w2, w3);
    }
}

// Merkle blocks (inputs.py gen_blocks): dst [batch][2^n][64] bytes = 8 LE64 words per block,
// word w of block x of tree I = splitmix64((I << 36) | (x << 3) | w).  One thread per word.
static __global__ void k_generate_blocks(uint64_t *dst, uint64_t batch, uint32_t n, uint64_t first_index,
                                         uint64_t seed) {
    const uint64_t words = batch << (n + 3);
    for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < words;
         e += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t xw = e & ((8ull << n) - 1), b = e >> (n + 3);
        dst[e] = splitmix64_ctr(((first_index + b) << 36) | xw, seed);
    }
}

}  // namespace bzk
