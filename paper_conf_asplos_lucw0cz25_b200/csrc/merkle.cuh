// merkle.cuh -- batched Merkle trees on B200 (readings R17-R19).
//
// A tree over N = 2^n 512-bit blocks (Sec. 3.1): level 0 = H(block_x) for every block, level
// l+1 [j] = H(level_l[2j] || level_l[2j+1]), root = level n [0]; 2N - 1 hashes.  H is one
// SHA-256 compression of the 512-bit block from the FIPS 180-4 IV ("produces a fixed-size
// 256-bit hash value from a 512-bit block", the default) or the full FIPS SHA-256 of the 64-byte
// message (a second compression of the constant padding block, whose schedule is folded into
// constants here).  The message words and the state stay in registers.
//
// Schedule (B200-first, not the paper's one-kernel-per-layer pipeline): a STAGE launch
// covers LT + 1 consecutive levels of every tree of the batch.  One thread owns 2^LT consecutive
// 64-byte blocks of one tree and hashes them plus every node above them up to its subtree root
// (2^(LT+1) - 1 hashes, one hash body in a loop, pending left siblings on a register stack): no
// barriers, no shared memory and no idle lanes.  The next stage reads those subtree roots as its
// blocks (two adjacent digests ARE the next 512-bit block), so a tree of 2^20 blocks takes
// ceil(21 / (LT + 1)) launches, each fully parallel over the whole batch; the paper's idle-thread
// problem of the upper layers (Fig. 4a) does not arise because every stage's threads are
// packed over all trees of the batch.
#pragma once
#include <stdint.h>

namespace bzk {
namespace mk {

// FIPS 180-4 Sec. 4.2.2 (K) and Sec. 5.3.3 (initial hash value)
#define BZK_MK_K                                                                                   \
    {0x428a2f98, 0x71374491, 0xb5c0fbcf, 0xe9b5dba5, 0x3956c25b, 0x59f111f1, 0x923f82a4, 0xab1c5ed5, \
     0xd807aa98, 0x12835b01, 0x243185be, 0x550c7dc3, 0x72be5d74, 0x80deb1fe, 0x9bdc06a7, 0xc19bf174, \
     0xe49b69c1, 0xefbe4786, 0x0fc19dc6, 0x240ca1cc, 0x2de92c6f, 0x4a7484aa, 0x5cb0a9dc, 0x76f988da, \
     0x983e5152, 0xa831c66d, 0xb00327c8, 0xbf597fc7, 0xc6e00bf3, 0xd5a79147, 0x06ca6351, 0x14292967, \
     0x27b70a85, 0x2e1b2138, 0x4d2c6dfc, 0x53380d13, 0x650a7354, 0x766a0abb, 0x81c2c92e, 0x92722c85, \
     0xa2bfe8a1, 0xa81a664b, 0xc24b8b70, 0xc76c51a3, 0xd192e819, 0xd6990624, 0xf40e3585, 0x106aa070, \
     0x19a4c116, 0x1e376c08, 0x2748774c, 0x34b0bcb5, 0x391c0cb3, 0x4ed8aa4a, 0x5b9cca4f, 0x682e6ff3, \
     0x748f82ee, 0x78a5636f, 0x84c87814, 0x8cc70208, 0x90befffa, 0xa4506ceb, 0xbef9a3f7, 0xc67178f2}

struct Tab64 { uint32_t v[64]; };

constexpr uint32_t crotr(uint32_t x, int n) { return (x >> n) | (x << (32 - n)); }

// K[t] + W[t] for the constant second block of a 64-byte message: 0x80 || 0^55 || BE64(512)
constexpr Tab64 make_pad_kw() {
    Tab64 k = {BZK_MK_K};
    uint32_t w[64] = {};
    w[0] = 0x80000000u;
    w[15] = 512u;
    for (int t = 16; t < 64; ++t) {
        uint32_t s0 = crotr(w[t - 15], 7) ^ crotr(w[t - 15], 18) ^ (w[t - 15] >> 3);
        uint32_t s1 = crotr(w[t - 2], 17) ^ crotr(w[t - 2], 19) ^ (w[t - 2] >> 10);
        w[t] = w[t - 16] + s0 + w[t - 7] + s1;
    }
    Tab64 r = {};
    for (int t = 0; t < 64; ++t) r.v[t] = k.v[t] + w[t];
    return r;
}

static __constant__ Tab64 c_K = {BZK_MK_K};
static __constant__ Tab64 c_pad_kw = make_pad_kw();

__device__ __forceinline__ uint32_t rotr(uint32_t x, int n) { return __funnelshift_r(x, x, n); }
__device__ __forceinline__ uint32_t bswap(uint32_t x) { return __byte_perm(x, 0, 0x0123); }

__device__ __forceinline__ void set_iv(uint32_t h[8]) {
    h[0] = 0x6a09e667u; h[1] = 0xbb67ae85u; h[2] = 0x3c6ef372u; h[3] = 0xa54ff53au;
    h[4] = 0x510e527fu; h[5] = 0x9b05688cu; h[6] = 0x1f83d9abu; h[7] = 0x5be0cd19u;
}

// Every addition is issued as IMAD (x * 1 + y, the 1 opaque to the compiler) on the FMA pipe,
// leaving the ALU pipe to the rotations and the logic (SHF, LOP3), which only it can execute:
// 6,366 -> 7,798 trees/s at 256 x 2^20 blocks.  K[t] + W[t] stays a plain add.
static __constant__ uint32_t c_one = 1;

__device__ __forceinline__ uint32_t fadd(uint32_t a, uint32_t b, uint32_t one) {
    uint32_t r;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(one), "r"(b));
    return r;
}

// One round with the working variables named by position (no register moves after unrolling).
#define BZK_MK_RND(a, b, c, d, e, f, g, h, kw)                                                     \
    do {                                                                                           \
        const uint32_t t1 = fadd(fadd(fadd(h, kw, one), (rotr(e, 6) ^ rotr(e, 11) ^ rotr(e, 25)), one), \
                                 ((e & f) ^ (~e & g)), one);                                        \
        d = fadd(d, t1, one);                                                                      \
        h = fadd(fadd(t1, (rotr(a, 2) ^ rotr(a, 13) ^ rotr(a, 22)), one), ((a & b) ^ (a & c) ^ (b & c)), one); \
    } while (0)

#define BZK_MK_8ROUNDS(T, KW)                         \
    BZK_MK_RND(a, b, c, d, e, f, g, h, KW(T + 0));    \
    BZK_MK_RND(h, a, b, c, d, e, f, g, KW(T + 1));    \
    BZK_MK_RND(g, h, a, b, c, d, e, f, KW(T + 2));    \
    BZK_MK_RND(f, g, h, a, b, c, d, e, KW(T + 3));    \
    BZK_MK_RND(e, f, g, h, a, b, c, d, KW(T + 4));    \
    BZK_MK_RND(d, e, f, g, h, a, b, c, KW(T + 5));    \
    BZK_MK_RND(c, d, e, f, g, h, a, b, KW(T + 6));    \
    BZK_MK_RND(b, c, d, e, f, g, h, a, KW(T + 7))

// The 64 rounds are fully unrolled (no moves to re-place the working variables).  With ONE hash body
// in the stage loop this no longer stalls on instruction fetch and beat a rolled 16-round body by 4 %
// (the first version inlined 8 unrolled bodies and did stall, ncu r01f).

// FIPS 180-4 Sec. 6.2.2: state st <- st + rounds(st, W); w[16] is the big-endian message (clobbered:
// it holds the rolling 16-word message schedule)
__device__ __forceinline__ void compress(uint32_t st[8], uint32_t w[16]) {
    const uint32_t one = c_one;
    uint32_t a = st[0], b = st[1], c = st[2], d = st[3], e = st[4], f = st[5], g = st[6], h = st[7];
#define BZK_MK_KW_MSG(t) (c_K.v[(t)] + w[(t) & 15])
#pragma unroll
    for (int T = 0; T < 64; T += 8) {
        if (T >= 16) {
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int t = T + j;
                const uint32_t w15 = w[(t - 15) & 15], w2 = w[(t - 2) & 15];
                w[t & 15] = fadd(fadd(fadd(w[t & 15], (rotr(w15, 7) ^ rotr(w15, 18) ^ (w15 >> 3)), one),
                                      w[(t - 7) & 15], one),
                                 (rotr(w2, 17) ^ rotr(w2, 19) ^ (w2 >> 10)), one);
            }
        }
        BZK_MK_8ROUNDS(T, BZK_MK_KW_MSG);
    }
#undef BZK_MK_KW_MSG
    st[0] += a; st[1] += b; st[2] += c; st[3] += d; st[4] += e; st[5] += f; st[6] += g; st[7] += h;
}

// compression of the constant padding block of a 64-byte message (schedule folded into c_pad_kw)
__device__ __forceinline__ void compress_pad64(uint32_t st[8]) {
    const uint32_t one = c_one;
    uint32_t a = st[0], b = st[1], c = st[2], d = st[3], e = st[4], f = st[5], g = st[6], h = st[7];
#define BZK_MK_KW_PAD(t) (c_pad_kw.v[(t)])
#pragma unroll
    for (int T = 0; T < 64; T += 8) { BZK_MK_8ROUNDS(T, BZK_MK_KW_PAD); }
#undef BZK_MK_KW_PAD
    st[0] += a; st[1] += b; st[2] += c; st[3] += d; st[4] += e; st[5] += f; st[6] += g; st[7] += h;
}

// H(512-bit block) -> digest words (big-endian state words).  MODE 0: one compression from the
// IV; MODE 1: FIPS SHA-256 of the 64-byte message (+ the constant padding block).
template <int MODE>
__device__ __forceinline__ void hash_block(uint32_t w[16], uint32_t out[8]) {
    set_iv(out);
    compress(out, w);
    if (MODE == 1) compress_pad64(out);
}

// ---------------------------------------------------------------- memory helpers (32-byte aligned)

__device__ __forceinline__ void ld_block(const uint8_t *p, uint32_t w[16]) {
    asm("ld.global.nc.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
        : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
        : "l"(p));
    asm("ld.global.nc.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8+32];"
        : "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]), "=r"(w[14]), "=r"(w[15])
        : "l"(p));
#pragma unroll
    for (int i = 0; i < 16; ++i) w[i] = bswap(w[i]);   // bytes -> big-endian message words
}

// digest words -> 32 bytes (big-endian words)
__device__ __forceinline__ void st_digest(uint8_t *p, const uint32_t h[8]) {
    asm volatile("st.global.v8.u32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(p), "r"(bswap(h[0])),
                 "r"(bswap(h[1])), "r"(bswap(h[2])), "r"(bswap(h[3])), "r"(bswap(h[4])), "r"(bswap(h[5])),
                 "r"(bswap(h[6])), "r"(bswap(h[7]))
                 : "memory");
}

// ---------------------------------------------------------------- stage kernel

struct StageParams {
    const uint8_t *in;          // this stage's 64-byte blocks; tree b at in + b * in_stride
    uint64_t in_stride;
    uint8_t *nodes;             // level-major node array [B][2N-1][32] or nullptr
    uint64_t nodes_stride;      // (2N - 1) * 32
    uint8_t *out;               // thread roots: out + b * out_stride + j * 32 (nullptr: not needed)
    uint64_t out_stride;
    uint64_t threads;           // B * 2^lg_tpt
    uint32_t n;                 // tree height (N = 2^n blocks)
    uint32_t lvl0;              // level of this stage's leaf hashes
    uint32_t lg_tpt;            // log2 threads per tree (= log2 M - LT)
};

// byte offset of node (level l, index j) in a tree's level-major node array
__device__ __forceinline__ uint64_t node_off(uint32_t n, uint32_t l, uint64_t j) {
    return (((2ull << n) - (2ull << (n - l))) + j) * 32ull;
}

// One thread = one subtree of 2^LT consecutive blocks of one tree: 2^(LT+1) - 1 hashes in post order
// (leaf, leaf, parent, leaf, leaf, parent, parent, ...), pending left siblings on a register stack,
// ONE hash body in the loop.  No barriers, no shared memory, no idle lanes: the levels above a
// thread root are the next stage's blocks.
template <int MODE, int LT>
__global__ void __launch_bounds__(256) k_merkle_stage(StageParams p) {
    const uint64_t gid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gid >= p.threads) return;
    const uint64_t b = gid >> p.lg_tpt;
    const uint64_t j0 = gid & ((1ull << p.lg_tpt) - 1);     // thread's subtree index within the tree
    const uint8_t *src = p.in + b * p.in_stride + (j0 << LT) * 64;
    uint8_t *nodes = p.nodes ? p.nodes + b * p.nodes_stride : nullptr;
    constexpr int L = 1 << LT;
    constexpr int SD = LT > 0 ? LT : 1;
    uint32_t stk[SD][8];        // stk[0] = most recently pushed left sibling
    uint32_t h[8];
    uint32_t leaf = 0, lvl = 0, pending = 0;
#pragma unroll 1
    for (int job = 0; job < 2 * L - 1; ++job) {
        uint32_t m[16];
        if (pending == 0) {
            ld_block(src + 64 * leaf, m);
        } else {
#pragma unroll
            for (int q = 0; q < 8; ++q) { m[q] = stk[0][q]; m[8 + q] = h[q]; }
#pragma unroll
            for (int s_ = 0; s_ + 1 < SD; ++s_)
#pragma unroll
                for (int q = 0; q < 8; ++q) stk[s_][q] = stk[s_ + 1][q];   // pop
        }
        hash_block<MODE>(m, h);
        if (pending == 0) {
            lvl = 0;
            pending = __ffs(~leaf) - 1;      // trailing one bits of the leaf index = merges to do now
            ++leaf;
        } else {
            ++lvl;
            --pending;
        }
        if (nodes) st_digest(nodes + node_off(p.n, p.lvl0 + lvl, ((j0 << LT) + leaf - 1) >> lvl), h);
        if (pending == 0 && job != 2 * L - 2) {
#pragma unroll
            for (int s_ = SD - 1; s_ > 0; --s_)
#pragma unroll
                for (int q = 0; q < 8; ++q) stk[s_][q] = stk[s_ - 1][q];   // push
#pragma unroll
            for (int q = 0; q < 8; ++q) stk[0][q] = h[q];
        }
    }
    if (p.out) st_digest(p.out + b * p.out_stride + j0 * 32, h);
}

}  // namespace mk

// k_merkle.cu: launch one stage (mode 0/1, per-thread subtree height lt in 0..4)
cudaError_t merkle_launch_stage(uint32_t mode, uint32_t lt, uint32_t grid, uint32_t threads, cudaStream_t s,
                                const mk::StageParams &p);

}  // namespace bzk
