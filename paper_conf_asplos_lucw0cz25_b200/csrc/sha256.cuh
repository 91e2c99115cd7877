// sha256.cuh -- FIPS 180-4 SHA-256 on the device, message schedule and state in registers
// (the paper keeps the 16 x 32-bit chunks in registers, Sec. 3.1).
//
// Transcript (reading R5-R7):
//   state_0 = SHA-256("BZK-SUMCHECK-V1\0" || seed || LE64 I || LE16 k || LE16 d || LE16 order || LE16 0)
//   state_i = SHA-256(state_{i-1} || LE256 g_i(0) || ... || LE256 g_i(d))
//   r_i     = LE256(state_i) mod p
// SHA-256 words are big-endian; field limbs are little-endian, so a LE256 limb enters the
// message schedule byte-swapped.
#pragma once
#include <stdint.h>
#include "field.cuh"

namespace bzk {

static __device__ __constant__ uint32_t c_K256[64] = {
    0x428a2f98, 0x71374491, 0xb5c0fbcf, 0xe9b5dba5, 0x3956c25b, 0x59f111f1, 0x923f82a4, 0xab1c5ed5,
    0xd807aa98, 0x12835b01, 0x243185be, 0x550c7dc3, 0x72be5d74, 0x80deb1fe, 0x9bdc06a7, 0xc19bf174,
    0xe49b69c1, 0xefbe4786, 0x0fc19dc6, 0x240ca1cc, 0x2de92c6f, 0x4a7484aa, 0x5cb0a9dc, 0x76f988da,
    0x983e5152, 0xa831c66d, 0xb00327c8, 0xbf597fc7, 0xc6e00bf3, 0xd5a79147, 0x06ca6351, 0x14292967,
    0x27b70a85, 0x2e1b2138, 0x4d2c6dfc, 0x53380d13, 0x650a7354, 0x766a0abb, 0x81c2c92e, 0x92722c85,
    0xa2bfe8a1, 0xa81a664b, 0xc24b8b70, 0xc76c51a3, 0xd192e819, 0xd6990624, 0xf40e3585, 0x106aa070,
    0x19a4c116, 0x1e376c08, 0x2748774c, 0x34b0bcb5, 0x391c0cb3, 0x4ed8aa4a, 0x5b9cca4f, 0x682e6ff3,
    0x748f82ee, 0x78a5636f, 0x84c87814, 0x8cc70208, 0x90befffa, 0xa4506ceb, 0xbef9a3f7, 0xc67178f2};

__device__ __forceinline__ uint32_t rotr32(uint32_t x, int n) { return __funnelshift_r(x, x, n); }
__device__ __forceinline__ uint32_t bswap32(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

__device__ __forceinline__ void sha256_init_state(uint32_t h[8]) {
    h[0] = 0x6a09e667; h[1] = 0xbb67ae85; h[2] = 0x3c6ef372; h[3] = 0xa54ff53a;
    h[4] = 0x510e527f; h[5] = 0x9b05688c; h[6] = 0x1f83d9ab; h[7] = 0x5be0cd19;
}

// one compression; w[16] = big-endian message words
__device__ __forceinline__ void sha256_compress(uint32_t h[8], const uint32_t win[16]) {
    uint32_t w[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) w[i] = win[i];
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4], f = h[5], g = h[6], hh = h[7];
#pragma unroll
    for (int t = 0; t < 64; ++t) {
        uint32_t wt;
        if (t < 16) {
            wt = w[t];
        } else {
            uint32_t w15 = w[(t - 15) & 15], w2 = w[(t - 2) & 15];
            uint32_t s0 = rotr32(w15, 7) ^ rotr32(w15, 18) ^ (w15 >> 3);
            uint32_t s1 = rotr32(w2, 17) ^ rotr32(w2, 19) ^ (w2 >> 10);
            wt = w[t & 15] + s0 + w[(t - 7) & 15] + s1;
            w[t & 15] = wt;
        }
        uint32_t S1 = rotr32(e, 6) ^ rotr32(e, 11) ^ rotr32(e, 25);
        uint32_t ch = (e & f) ^ (~e & g);
        uint32_t T1 = hh + S1 + ch + c_K256[t] + wt;
        uint32_t S0 = rotr32(a, 2) ^ rotr32(a, 13) ^ rotr32(a, 22);
        uint32_t maj = (a & b) ^ (a & c) ^ (b & c);
        hh = g; g = f; f = e; e = d + T1; d = c; c = b; b = a; a = T1 + S0 + maj;
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e; h[5] += f; h[6] += g; h[7] += hh;
}

// The same compression for the SERIAL per-round transcript (one thread per proof, on the critical path
// of every round): one NON-inlined, fully unrolled copy (K as immediates, no loop overhead) shared by
// every call site, instead of three inlined copies per transcript (which thrashed the instruction
// cache: k_small was 22K SASS instructions, ncu no_instruction stalls).
static __device__ __noinline__ void sha256_compress_serial(uint32_t h[8], const uint32_t win[16]) {
    uint32_t w[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) w[i] = win[i];
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4], f = h[5], g = h[6], hh = h[7];
#pragma unroll
    for (int T = 0; T < 64; T += 16) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            uint32_t wt;
            if (T == 0) {
                wt = w[j];
            } else {
                const uint32_t w15 = w[(j + 1) & 15], w2 = w[(j + 14) & 15];
                const uint32_t s0 = rotr32(w15, 7) ^ rotr32(w15, 18) ^ (w15 >> 3);
                const uint32_t s1 = rotr32(w2, 17) ^ rotr32(w2, 19) ^ (w2 >> 10);
                wt = w[j] + s0 + w[(j + 9) & 15] + s1;
                w[j] = wt;
            }
            const uint32_t S1 = rotr32(e, 6) ^ rotr32(e, 11) ^ rotr32(e, 25);
            const uint32_t ch = (e & f) ^ (~e & g);
            const uint32_t T1 = hh + S1 + ch + c_K256[T + j] + wt;
            const uint32_t S0 = rotr32(a, 2) ^ rotr32(a, 13) ^ rotr32(a, 22);
            const uint32_t maj = (a & b) ^ (a & c) ^ (b & c);
            hh = g; g = f; f = e; e = d + T1; d = c; c = b; b = a; a = T1 + S0 + maj;
        }
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e; h[5] += f; h[6] += g; h[7] += hh;
}

// Streaming absorber over 32-bit big-endian words (messages here are multiples of 4 bytes).
struct sha256_words {
    uint32_t h[8];
    uint32_t buf[16];
    uint32_t n;       // words in buf
    uint32_t total;   // total words absorbed
    __device__ __forceinline__ void init() { sha256_init_state(h); n = 0; total = 0; }
    __device__ __forceinline__ void push(uint32_t w) {
        // buf index is dynamic: keep it in local memory (this runs once per proof per round)
        buf[n++] = w;
        ++total;
        if (n == 16) { sha256_compress(h, buf); n = 0; }
    }
    __device__ __forceinline__ void finish(uint32_t out[8]) {
        uint64_t bits = (uint64_t)total * 32;
        push(0x80000000u);
        --total;  // padding does not count
        while (n != 14) { buf[n++] = 0; if (n == 16) { sha256_compress(h, buf); n = 0; } }
        buf[14] = (uint32_t)(bits >> 32);
        buf[15] = (uint32_t)bits;
        sha256_compress(h, buf);
#pragma unroll
        for (int i = 0; i < 8; ++i) out[i] = h[i];
    }
};

// digest words (big-endian H0..H7) -> LE256 integer limbs (limb j = bswap(H_j))
__device__ __forceinline__ fe digest_to_fe_raw(const uint32_t s[8]) {
    fe r;
#pragma unroll
    for (int i = 0; i < 8; ++i) r.l[i] = bswap32(s[i]);
    return r;
}

// state_0 for proof I (64-byte init block + 1 padding block)
// field_id: 0 = BN254 Fr, 1 = Goldilocks (reading R15; the last LE16 of the init block)
__device__ __forceinline__ void transcript_init(uint32_t state[8], const uint8_t seed[32], uint64_t I,
                                                uint32_t k, uint32_t d, uint32_t order, uint32_t field_id = 0) {
    sha256_words sh;
    sh.init();
    // "BZK-SUMCHECK-V1\0" as big-endian words
    sh.push(0x425a4b2du);  // "BZK-"
    sh.push(0x53554d43u);  // "SUMC"
    sh.push(0x4845434bu);  // "HECK"
    sh.push(0x2d563100u);  // "-V1\0"
#pragma unroll
    for (int i = 0; i < 8; ++i)
        sh.push(((uint32_t)seed[4 * i] << 24) | ((uint32_t)seed[4 * i + 1] << 16) |
                ((uint32_t)seed[4 * i + 2] << 8) | (uint32_t)seed[4 * i + 3]);
    sh.push(bswap32((uint32_t)I));
    sh.push(bswap32((uint32_t)(I >> 32)));
    sh.push(bswap32((k & 0xffffu) | ((d & 0xffffu) << 16)));
    sh.push(bswap32((order & 0xffffu) | ((field_id & 0xffffu) << 16)));
    sh.finish(state);
}

// state_i = SHA-256(state_{i-1} || LE256 g(0..D)) with the message laid out at compile time: the
// 8 + 8 (D + 1) words, the 0x80 marker, zeros and the 64-bit length sit in a static word array, so
// every block is compressed straight from registers (no streaming buffer in local memory).  This is
// the serial part of every round (one thread per proof), so its latency is what counts.
template <int D>
__device__ __forceinline__ fe transcript_round_t(uint32_t state[8], const fe (&g)[D + 1]) {
    constexpr int N = 8 + 8 * (D + 1);                  // message words
    constexpr int NB = (N + 1 + 2 + 15) / 16;           // blocks incl. the marker and the length
    uint32_t m[NB * 16];
#pragma unroll
    for (int i = 0; i < 8; ++i) m[i] = state[i];
#pragma unroll
    for (int t = 0; t <= D; ++t)
#pragma unroll
        for (int i = 0; i < 8; ++i) m[8 + 8 * t + i] = bswap32(g[t].l[i]);
    m[N] = 0x80000000u;
#pragma unroll
    for (int i = N + 1; i < NB * 16 - 2; ++i) m[i] = 0;
    m[NB * 16 - 2] = 0;
    m[NB * 16 - 1] = (uint32_t)N * 32;
    uint32_t h[8];
    sha256_init_state(h);
#pragma unroll 1
    for (int b = 0; b < NB; ++b) sha256_compress_serial(h, m + 16 * b);
#pragma unroll
    for (int i = 0; i < 8; ++i) state[i] = h[i];
    return fe_reduce_256(digest_to_fe_raw(state));
}

// state_i = SHA-256(state_{i-1} || LE256 g(0..d)); returns r_i canonical (standard form)
__device__ __forceinline__ fe transcript_round(uint32_t state[8], const fe *g, int d) {
    sha256_words sh;
    sh.init();
#pragma unroll 1
    for (int i = 0; i < 8; ++i) sh.push(state[i]);
#pragma unroll 1
    for (int t = 0; t <= d; ++t)
#pragma unroll 1
        for (int i = 0; i < 8; ++i) sh.push(bswap32(g[t].l[i]));
    sh.finish(state);
    return fe_reduce_256(digest_to_fe_raw(state));
}

}  // namespace bzk
