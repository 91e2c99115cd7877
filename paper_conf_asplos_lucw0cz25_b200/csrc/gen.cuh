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

// Range bounds of the generated values (the moduli as raw words; the only "field" content here):
// a value drawn from [0, 2^254) that lands in [p, 2^254) is moved down by p once (inputs.py).
__device__ __constant__ const uint64_t kGenP[4] = {0x43E1F593F0000001ull, 0x2833E84879B97091ull,
                                                    0xB85045B68181585Dull, 0x30644E72E131A029ull};
constexpr uint64_t kGenPgl = 0xFFFFFFFF00000001ull;
constexpr uint64_t kAdvTableSalt = 0x5441424C45414456ull;   // "TABLEADV"
constexpr uint64_t kAdvElemSalt = 0x454C454D41445653ull;    // "ELEMADVS"

__device__ __forceinline__ void gen_canonical_254(uint64_t w[4]) {
    w[3] &= (1ull << 62) - 1;
    bool ge = true;                                    // w >= p, decided from the top limb down
    for (int i = 3; i >= 0; --i) {
        if (w[i] != kGenP[i]) { ge = w[i] > kGenP[i]; break; }
    }
    if (ge) {
        uint64_t borrow = 0;
        for (int i = 0; i < 4; ++i) {
            const uint64_t pi = kGenP[i];
            const uint64_t r = w[i] - pi - borrow;
            borrow = (w[i] < pi || (w[i] == pi && borrow)) ? 1 : 0;
            w[i] = r;
        }
    }
}

// adversarial modes (inputs.py _adv_modes): table mode = word'(I, m) mod 5; mode 4 -> per element
__device__ __forceinline__ void gen_adv_mode(uint64_t base, uint64_t x, uint64_t seed, int &tmode, int &mode) {
    tmode = (int)(splitmix64_ctr(base, seed ^ kAdvTableSalt) % 5);
    mode = tmode < 4 ? tmode : (int)(splitmix64_ctr(base | (x << 2), seed ^ kAdvElemSalt) % 5);
}

// dst: [batch][d][2^k][4] u64; one thread per element (4 words, stored as 2 x 16 B)
// dist 0 uniform, 1 smallint, 2 vml, 3 Goldilocks (one word), 4 adversarial, 5 Goldilocks adversarial
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
        if (dist == 3 || dist == 5) {   // Goldilocks: one word per element
            const uint64_t w = splitmix64_ctr(base, seed);
            uint64_t v = w >= kGenPgl ? w - kGenPgl : w;
            if (dist == 5) {
                int tmode, mode;
                gen_adv_mode((I << 36) | (m << 32), x, seed, tmode, mode);
                if (mode == 0) v = kGenPgl - 1 - (w & 0xffffull);
                else if (mode == 1) v = kGenPgl - 1;
                else if (mode == 2) v = (tmode == 4 || (x & 1) == 0) ? 0 : kGenPgl - 1;
                else if (mode == 3) v = (w & ((1ull << 62) - 1)) | (1ull << 63);
            }
            dst[e] = v;
            continue;
        }
        bool small = dist == 1 || (dist == 2 && m == 0);
        uint64_t w[4];
        if (small) {
            w[0] = splitmix64_ctr(base, seed) & 0xffull;
            w[1] = w[2] = w[3] = 0;
        } else {
            uint64_t raw[4];
            for (int i = 0; i < 4; ++i) raw[i] = w[i] = splitmix64_ctr(base | i, seed);
            gen_canonical_254(w);
            if (dist == 4) {
                int tmode, mode;
                gen_adv_mode((I << 36) | (m << 32), x, seed, tmode, mode);
                uint64_t pm1[4] = {kGenP[0] - 1, kGenP[1], kGenP[2], kGenP[3]};
                if (mode == 0) {
                    for (int i = 0; i < 4; ++i) w[i] = pm1[i];
                    w[0] -= raw[0] & 0xffffull;
                } else if (mode == 1 || mode == 2) {
                    const bool zero = mode == 2 && (tmode == 4 || (x & 1) == 0);
                    for (int i = 0; i < 4; ++i) w[i] = zero ? 0 : pm1[i];
                } else if (mode == 3) {
                    for (int i = 0; i < 3; ++i) w[i] = raw[i];
                    w[3] = (raw[3] & ((1ull << 60) - 1)) | (1ull << 61);
                }
            }
        }
        ulonglong2 *q = reinterpret_cast<ulonglong2 *>(dst + 4 * e);
        q[0] = make_ulonglong2(w[0], w[1]);
        q[1] = make_ulonglong2(w[2], w[3]);
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
