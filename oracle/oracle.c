/*
 * oracle/oracle.c -- CPU ORACLE for the batched sum-check prover.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path may include, link,
 * load or call this file: only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference leg use it.  It shares no code, header,
 * constant table or helper with the CUDA path (paper_conf_asplos_lucw0cz25_b200/csrc).
 *
 * It is deliberately plain and slow:
 *   - field elements are 4 x u64 little-endian limbs, always canonical (< p);
 *   - a*b mod p is a schoolbook 512-bit product (unsigned __int128) followed by
 *     Barrett reduction (Menezes/van Oorschot/Vanstone, HAC Alg. 14.42) with
 *     mu = floor(2^512 / p) computed at start-up by bit-serial long division;
 *   - no Montgomery form, no lazy reduction, no fusion: every step follows the
 *     paper's Algorithm 1 (Sec. 2.3) generalised as written
 *     in SURVEY.md Sec. 8(c.2) / DESIGN.md "Readings".
 *
 * What each function follows (P:L = /root/reference/PAPER.md line L):
 *   orc_prove    -- SURVEY 8(c.2) steps 1-5: per round i, g_i(t) for t = 0..d
 *                   (Alg.1 lines 3-4 generalised to a product of d
 *                   multilinears), Fiat-Shamir challenge from SHA-256 (P:97,
 *                   P:211; reading R5-R7), fold A <- A + r(A' - A)
 *                   (P:111 line 5, reading R8).
 *   orc_alg1     -- P:111 Algorithm 1 literally (d = 1, pairs (b, b+2^{n-i}),
 *                   update (1-r)A[b] + r A[b+2^{n-i}], r_i given as input).
 *   orc_verify   -- the O(n) verifier of P:101.
 *   orc_mle      -- multilinear extension f(rho) = sum_x T[x] eq(x, rho), the
 *                   plain definition (independent of folding).
 *   orc_hsum     -- H = sum_{x in {0,1}^k} prod_m T_m[x].
 *   orc_sha256   -- FIPS 180-4 SHA-256 (the paper's hash).
 *   orc_merkle   -- Merkle tree of N = 2^n 512-bit blocks, level by level as
 *                   P:91-97 (Sec. 2.2, Fig. 2) describes it; H = one SHA-256
 *                   compression of the block (reading R18) or full
 *                   FIPS SHA-256; orc_merkle_path / orc_merkle_verify_path
 *                   open and check one leaf ("efficient verifiability").
 *   orc_encode   -- Spielman-style linear-time encoder, recursively as P:113-117
 *                   (Sec. 2.4, Fig. 3) describes it; graphs are inputs (R21-R24).
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"): Python exact integers for the
 * field, FIPS 180-4 vectors + hashlib for SHA-256, brute-force hypercube sums,
 * the round invariant g_i(0)+g_i(1) = g_{i-1}(r_{i-1}), the degree pin at
 * t = d+1, final_m = MLE(T_m)(rho) via eq-tables, closed forms, Alg.1 literal
 * mode, an independent Python cross-oracle, and verifier mutation tests.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

typedef unsigned __int128 u128;
typedef struct { uint64_t v[4]; } fr;

/* BN254 scalar field modulus r (reading R1): 0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001 */
static const fr P = {{0x43e1f593f0000001ULL, 0x2833e84879b97091ULL,
                      0xb85045b68181585dULL, 0x30644e72e131a029ULL}};
static uint64_t MU[5];           /* floor(2^512 / p), 259 bits */
static int mu_ready = 0;
static pthread_mutex_t mu_lock = PTHREAD_MUTEX_INITIALIZER;

/* ------------------------------------------------------------------ */
/* multi-precision helpers (plain)                                     */
/* ------------------------------------------------------------------ */

/* compare two n-limb numbers: -1, 0, 1 */
static int mp_cmp(const uint64_t *a, const uint64_t *b, int n) {
    for (int i = n - 1; i >= 0; --i) {
        if (a[i] < b[i]) return -1;
        if (a[i] > b[i]) return 1;
    }
    return 0;
}

/* r = a - b over n limbs, returns borrow */
static uint64_t mp_sub(uint64_t *r, const uint64_t *a, const uint64_t *b, int n) {
    uint64_t borrow = 0;
    for (int i = 0; i < n; ++i) {
        u128 d = (u128)a[i] - b[i] - borrow;
        r[i] = (uint64_t)d;
        borrow = (uint64_t)(d >> 64) ? 1 : 0;
    }
    return borrow;
}

/* r = a + b over n limbs, returns carry */
static uint64_t mp_add(uint64_t *r, const uint64_t *a, const uint64_t *b, int n) {
    uint64_t carry = 0;
    for (int i = 0; i < n; ++i) {
        u128 s = (u128)a[i] + b[i] + carry;
        r[i] = (uint64_t)s;
        carry = (uint64_t)(s >> 64);
    }
    return carry;
}

/* r[0..na+nb) = a[0..na) * b[0..nb)  (schoolbook) */
static void mp_mul(uint64_t *r, const uint64_t *a, int na, const uint64_t *b, int nb) {
    for (int i = 0; i < na + nb; ++i) r[i] = 0;
    for (int i = 0; i < na; ++i) {
        uint64_t carry = 0;
        for (int j = 0; j < nb; ++j) {
            u128 t = (u128)a[i] * b[j] + r[i + j] + carry;
            r[i + j] = (uint64_t)t;
            carry = (uint64_t)(t >> 64);
        }
        r[i + nb] = carry;
    }
}

/* mu = floor(2^512 / p) by bit-serial long division (slow, once). */
static void compute_mu(void) {
    uint64_t rem[5] = {0, 0, 0, 0, 0};   /* remainder < p < 2^254, 2*rem fits */
    uint64_t q[9] = {0};                 /* quotient bits 0..512 */
    uint64_t p5[5] = {P.v[0], P.v[1], P.v[2], P.v[3], 0};
    for (int bit = 512; bit >= 0; --bit) {
        /* rem = 2*rem + (bit of 2^512) */
        for (int i = 4; i > 0; --i) rem[i] = (rem[i] << 1) | (rem[i - 1] >> 63);
        rem[0] <<= 1;
        if (bit == 512) rem[0] |= 1;
        if (mp_cmp(rem, p5, 5) >= 0) {
            mp_sub(rem, rem, p5, 5);
            q[bit / 64] |= (uint64_t)1 << (bit % 64);
        }
    }
    for (int i = 0; i < 5; ++i) MU[i] = q[i];
}

static void ensure_mu(void) {
    if (__atomic_load_n(&mu_ready, __ATOMIC_ACQUIRE)) return;
    pthread_mutex_lock(&mu_lock);
    if (!mu_ready) { compute_mu(); __atomic_store_n(&mu_ready, 1, __ATOMIC_RELEASE); }
    pthread_mutex_unlock(&mu_lock);
}

/* ------------------------------------------------------------------ */
/* field F_p                                                            */
/* ------------------------------------------------------------------ */

static int fr_is_canon(const fr *a) { return mp_cmp(a->v, P.v, 4) < 0; }

static fr fr_zero(void) { fr z = {{0, 0, 0, 0}}; return z; }
static fr fr_from_u64(uint64_t x) { fr z = {{x, 0, 0, 0}}; return z; }
static int fr_eq(const fr *a, const fr *b) { return mp_cmp(a->v, b->v, 4) == 0; }

static fr fr_add(fr a, fr b) {
    fr r;
    uint64_t c = mp_add(r.v, a.v, b.v, 4);
    /* a, b < p < 2^254 so no carry out of 256 bits; subtract p once if needed */
    if (c || mp_cmp(r.v, P.v, 4) >= 0) mp_sub(r.v, r.v, P.v, 4);
    return r;
}

static fr fr_sub(fr a, fr b) {
    fr r;
    uint64_t borrow = mp_sub(r.v, a.v, b.v, 4);
    if (borrow) mp_add(r.v, r.v, P.v, 4);
    return r;
}

/* x (8 limbs, x < 2^512) mod p: Barrett, HAC Alg. 14.42 with b = 2^64, k = 4 */
static fr barrett_reduce(const uint64_t x[8]) {
    uint64_t q1[5], q2[10], q3[5], r1[5], r2full[10], r2[5], r[5];
    for (int i = 0; i < 5; ++i) q1[i] = x[3 + i];          /* floor(x / b^{k-1}) */
    mp_mul(q2, q1, 5, MU, 5);                               /* q1 * mu */
    for (int i = 0; i < 5; ++i) q3[i] = q2[5 + i];          /* floor(q2 / b^{k+1}) */
    for (int i = 0; i < 5; ++i) r1[i] = x[i];               /* x mod b^{k+1} */
    uint64_t p5[5] = {P.v[0], P.v[1], P.v[2], P.v[3], 0};
    mp_mul(r2full, q3, 5, p5, 5);
    for (int i = 0; i < 5; ++i) r2[i] = r2full[i];          /* q3*p mod b^{k+1} */
    mp_sub(r, r1, r2, 5);                                   /* mod b^{k+1} (wraps) */
    while (mp_cmp(r, p5, 5) >= 0) mp_sub(r, r, p5, 5);     /* at most twice */
    fr out = {{r[0], r[1], r[2], r[3]}};
    return out;
}

static fr fr_mul(fr a, fr b) {
    uint64_t x[8];
    mp_mul(x, a.v, 4, b.v, 4);
    return barrett_reduce(x);
}

static fr fr_pow(fr a, const uint64_t e[4]) {
    fr r = fr_from_u64(1);
    for (int i = 255; i >= 0; --i) {
        r = fr_mul(r, r);
        if ((e[i / 64] >> (i % 64)) & 1) r = fr_mul(r, a);
    }
    return r;
}

/* a^{-1} = a^{p-2} (Fermat); a != 0 */
static fr fr_inv(fr a) {
    uint64_t e[4] = {P.v[0] - 2, P.v[1], P.v[2], P.v[3]};
    return fr_pow(a, e);
}

/* reduce an arbitrary 256-bit integer mod p (for hash -> field, reading R7) */
static fr fr_from_256(const uint64_t v[4]) {
    uint64_t x[8] = {v[0], v[1], v[2], v[3], 0, 0, 0, 0};
    return barrett_reduce(x);
}

/* ------------------------------------------------------------------ */
/* SHA-256, FIPS 180-4                                                  */
/* ------------------------------------------------------------------ */

typedef struct { uint32_t h[8]; uint8_t buf[64]; uint64_t len; uint32_t nbuf; } sha256_ctx;

static const uint32_t K256[64] = {
    0x428a2f98, 0x71374491, 0xb5c0fbcf, 0xe9b5dba5, 0x3956c25b, 0x59f111f1, 0x923f82a4, 0xab1c5ed5,
    0xd807aa98, 0x12835b01, 0x243185be, 0x550c7dc3, 0x72be5d74, 0x80deb1fe, 0x9bdc06a7, 0xc19bf174,
    0xe49b69c1, 0xefbe4786, 0x0fc19dc6, 0x240ca1cc, 0x2de92c6f, 0x4a7484aa, 0x5cb0a9dc, 0x76f988da,
    0x983e5152, 0xa831c66d, 0xb00327c8, 0xbf597fc7, 0xc6e00bf3, 0xd5a79147, 0x06ca6351, 0x14292967,
    0x27b70a85, 0x2e1b2138, 0x4d2c6dfc, 0x53380d13, 0x650a7354, 0x766a0abb, 0x81c2c92e, 0x92722c85,
    0xa2bfe8a1, 0xa81a664b, 0xc24b8b70, 0xc76c51a3, 0xd192e819, 0xd6990624, 0xf40e3585, 0x106aa070,
    0x19a4c116, 0x1e376c08, 0x2748774c, 0x34b0bcb5, 0x391c0cb3, 0x4ed8aa4a, 0x5b9cca4f, 0x682e6ff3,
    0x748f82ee, 0x78a5636f, 0x84c87814, 0x8cc70208, 0x90befffa, 0xa4506ceb, 0xbef9a3f7, 0xc67178f2};

static uint32_t rotr(uint32_t x, int n) { return (x >> n) | (x << (32 - n)); }

static void sha256_block(uint32_t h[8], const uint8_t blk[64]) {
    uint32_t w[64];
    for (int t = 0; t < 16; ++t)
        w[t] = ((uint32_t)blk[4 * t] << 24) | ((uint32_t)blk[4 * t + 1] << 16) |
               ((uint32_t)blk[4 * t + 2] << 8) | (uint32_t)blk[4 * t + 3];
    for (int t = 16; t < 64; ++t) {
        uint32_t s0 = rotr(w[t - 15], 7) ^ rotr(w[t - 15], 18) ^ (w[t - 15] >> 3);
        uint32_t s1 = rotr(w[t - 2], 17) ^ rotr(w[t - 2], 19) ^ (w[t - 2] >> 10);
        w[t] = w[t - 16] + s0 + w[t - 7] + s1;
    }
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4], f = h[5], g = h[6], hh = h[7];
    for (int t = 0; t < 64; ++t) {
        uint32_t S1 = rotr(e, 6) ^ rotr(e, 11) ^ rotr(e, 25);
        uint32_t ch = (e & f) ^ (~e & g);
        uint32_t T1 = hh + S1 + ch + K256[t] + w[t];
        uint32_t S0 = rotr(a, 2) ^ rotr(a, 13) ^ rotr(a, 22);
        uint32_t maj = (a & b) ^ (a & c) ^ (b & c);
        uint32_t T2 = S0 + maj;
        hh = g; g = f; f = e; e = d + T1; d = c; c = b; b = a; a = T1 + T2;
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e; h[5] += f; h[6] += g; h[7] += hh;
}

static void sha256_init(sha256_ctx *c) {
    static const uint32_t H0[8] = {0x6a09e667, 0xbb67ae85, 0x3c6ef372, 0xa54ff53a,
                                   0x510e527f, 0x9b05688c, 0x1f83d9ab, 0x5be0cd19};
    memcpy(c->h, H0, sizeof H0);
    c->len = 0; c->nbuf = 0;
}

static void sha256_update(sha256_ctx *c, const uint8_t *m, size_t n) {
    for (size_t i = 0; i < n; ++i) {
        c->buf[c->nbuf++] = m[i];
        if (c->nbuf == 64) { sha256_block(c->h, c->buf); c->nbuf = 0; }
    }
    c->len += n;
}

static void sha256_final(sha256_ctx *c, uint8_t out[32]) {
    uint64_t bits = c->len * 8;
    uint8_t one = 0x80, zero = 0;
    sha256_update(c, &one, 1);
    while (c->nbuf != 56) sha256_update(c, &zero, 1);
    uint8_t lenb[8];
    for (int i = 0; i < 8; ++i) lenb[i] = (uint8_t)(bits >> (56 - 8 * i));
    sha256_update(c, lenb, 8);
    for (int i = 0; i < 8; ++i) {
        out[4 * i] = (uint8_t)(c->h[i] >> 24); out[4 * i + 1] = (uint8_t)(c->h[i] >> 16);
        out[4 * i + 2] = (uint8_t)(c->h[i] >> 8); out[4 * i + 3] = (uint8_t)c->h[i];
    }
}

void orc_sha256(const uint8_t *msg, uint64_t len, uint8_t out[32]) {
    sha256_ctx c; sha256_init(&c); sha256_update(&c, msg, (size_t)len); sha256_final(&c, out);
}

/* ------------------------------------------------------------------ */
/* transcript (reading R5-R7)            */
/* ------------------------------------------------------------------ */

static void le_bytes_of_fr(const fr *a, uint8_t out[32]) {
    for (int i = 0; i < 4; ++i)
        for (int j = 0; j < 8; ++j) out[8 * i + j] = (uint8_t)(a->v[i] >> (8 * j));
}

static fr fr_of_le_bytes_mod_p(const uint8_t in[32]) {
    uint64_t v[4] = {0, 0, 0, 0};
    for (int i = 0; i < 4; ++i)
        for (int j = 0; j < 8; ++j) v[i] |= (uint64_t)in[8 * i + j] << (8 * j);
    return fr_from_256(v);
}

/* state_0 = SHA-256("BZK-SUMCHECK-V1\0" || seed || LE64(I) || LE16 k || LE16 d || LE16 order || LE16 0) */
static void transcript_init(uint8_t state[32], const uint8_t seed[32], uint64_t I,
                            uint32_t k, uint32_t d, uint32_t order) {
    uint8_t m[64];
    memcpy(m, "BZK-SUMCHECK-V1", 15); m[15] = 0;
    memcpy(m + 16, seed, 32);
    for (int i = 0; i < 8; ++i) m[48 + i] = (uint8_t)(I >> (8 * i));
    m[56] = (uint8_t)k; m[57] = (uint8_t)(k >> 8);
    m[58] = (uint8_t)d; m[59] = (uint8_t)(d >> 8);
    m[60] = (uint8_t)order; m[61] = (uint8_t)(order >> 8);
    m[62] = 0; m[63] = 0;
    orc_sha256(m, 64, state);
}

/* state_i = SHA-256(state_{i-1} || LE256 g(0) || ... || LE256 g(d)); r_i = LE(state_i) mod p */
static fr transcript_round(uint8_t state[32], const fr *g, uint32_t d) {
    sha256_ctx c; sha256_init(&c);
    sha256_update(&c, state, 32);
    for (uint32_t t = 0; t <= d; ++t) { uint8_t b[32]; le_bytes_of_fr(&g[t], b); sha256_update(&c, b, 32); }
    sha256_final(&c, state);
    return fr_of_le_bytes_mod_p(state);
}

/* ------------------------------------------------------------------ */
/* prover                                                */
/* ------------------------------------------------------------------ */

enum { ORC_OK = 0, ORC_EINVAL = 1, ORC_ENONCANON = 4, ORC_ENOMEM = 2 };

/*
 * One proof.  tables: [d][2^k] elements, each 4 u64 LE canonical; never mutated.
 * round_evals: [k][d+1][4]; challenges: [k][4]; final_evals: [d][4]; claim: [4] (may be NULL).
 * order 0 = LSB (pairs (2j, 2j+1), binds x_1 first); 1 = MSB (pairs (j, j+h), Alg. 1).
 */
static int prove_impl(uint32_t k, uint32_t d, uint32_t order, const uint8_t seed[32], uint64_t I,
                      const uint64_t *tables, uint64_t *round_evals, uint64_t *challenges,
                      uint64_t *final_evals, uint64_t *claim, const uint64_t *given_r) {
    if (k > 30 || d < 1 || d > 4 || order > 1) return ORC_EINVAL;
    ensure_mu();
    const uint64_t N = (uint64_t)1 << k;
    /* step 2: copy the tables (never mutate the input) */
    fr *T = (fr *)malloc(sizeof(fr) * N * d);
    if (!T) return ORC_ENOMEM;
    for (uint64_t x = 0; x < N * d; ++x) {
        memcpy(T[x].v, tables + 4 * x, 32);
        if (!fr_is_canon(&T[x])) { free(T); return ORC_ENONCANON; }
    }
    /* H = sum_x prod_m T_m[x] -- brute force, emitted as the claim */
    fr H = fr_zero();
    for (uint64_t x = 0; x < N; ++x) {
        fr prod = T[x];
        for (uint32_t m = 1; m < d; ++m) prod = fr_mul(prod, T[m * N + x]);
        H = fr_add(H, prod);
    }
    /* step 1: transcript */
    uint8_t state[32];
    transcript_init(state, seed, I, k, d, order);
    /* step 3: rounds */
    uint64_t size = N;                              /* current table size per m */
    fr g[5];
    for (uint32_t i = 1; i <= k; ++i) {
        uint64_t h = size / 2;                       /* h = 2^{k-i} */
        /* (a) g_i(t) = sum_j prod_m (a_mj + t (b_mj - a_mj)), t = 0..d */
        for (uint32_t t = 0; t <= d; ++t) {
            fr tt = fr_from_u64(t);
            fr acc = fr_zero();
            for (uint64_t j = 0; j < h; ++j) {
                fr prod = fr_from_u64(1);
                for (uint32_t m = 0; m < d; ++m) {
                    fr *Tm = T + (uint64_t)m * N;
                    fr a = order == 0 ? Tm[2 * j] : Tm[j];
                    fr b = order == 0 ? Tm[2 * j + 1] : Tm[j + h];
                    fr v = fr_add(a, fr_mul(tt, fr_sub(b, a)));
                    prod = fr_mul(prod, v);
                }
                acc = fr_add(acc, prod);
            }
            g[t] = acc;
        }
        /* (b), (c) transcript -> r_i; or, paper-literal mode (Alg. 1), r_i given */
        fr r;
        if (given_r) {
            memcpy(r.v, given_r + 4 * (uint64_t)(i - 1), 32);
            if (!fr_is_canon(&r)) { free(T); return ORC_ENONCANON; }
        } else {
            r = transcript_round(state, g, d);
        }
        for (uint32_t t = 0; t <= d; ++t)
            memcpy(round_evals + 4 * ((uint64_t)(i - 1) * (d + 1) + t), g[t].v, 32);
        memcpy(challenges + 4 * (uint64_t)(i - 1), r.v, 32);
        /* (d) fold: T_m[j] := a + r (b - a), new size h */
        for (uint32_t m = 0; m < d; ++m) {
            fr *Tm = T + (uint64_t)m * N;
            for (uint64_t j = 0; j < h; ++j) {
                fr a = order == 0 ? Tm[2 * j] : Tm[j];
                fr b = order == 0 ? Tm[2 * j + 1] : Tm[j + h];
                Tm[j] = fr_add(a, fr_mul(r, fr_sub(b, a)));
            }
        }
        size = h;
    }
    /* step 4 / 5 */
    for (uint32_t m = 0; m < d; ++m) memcpy(final_evals + 4 * m, T[(uint64_t)m * N].v, 32);
    if (claim) memcpy(claim, H.v, 32);
    free(T);
    return ORC_OK;
}

int orc_prove(uint32_t k, uint32_t d, uint32_t order, const uint8_t seed[32], uint64_t I,
              const uint64_t *tables, uint64_t *round_evals, uint64_t *challenges,
              uint64_t *final_evals, uint64_t *claim) {
    return prove_impl(k, d, order, seed, I, tables, round_evals, challenges, final_evals, claim, NULL);
}

/* Paper-literal mode: challenges r_1..r_k are inputs (Alg. 1), no transcript.  The same
 * fold algorithm; `challenges` is read and copied through unchanged. */
int orc_prove_given(uint32_t k, uint32_t d, uint32_t order, const uint64_t *tables, const uint64_t *given_r,
                    uint64_t *round_evals, uint64_t *challenges_out, uint64_t *final_evals, uint64_t *claim) {
    uint8_t seed[32] = {0};
    return prove_impl(k, d, order, seed, 0, tables, round_evals, challenges_out, final_evals, claim, given_r);
}

/* batch of proofs over pthreads (one proof per task) */
typedef struct {
    uint32_t k, d, order; const uint8_t *seed; uint64_t first_index, batch;
    const uint64_t *tables; uint64_t *round_evals, *challenges, *final_evals, *claims;
    uint64_t next; pthread_mutex_t lock; int status;
} batch_job;

static void *batch_worker(void *arg) {
    batch_job *j = (batch_job *)arg;
    const uint64_t N = (uint64_t)1 << j->k;
    for (;;) {
        pthread_mutex_lock(&j->lock);
        uint64_t b = j->next++;
        pthread_mutex_unlock(&j->lock);
        if (b >= j->batch) break;
        int s = orc_prove(j->k, j->d, j->order, j->seed, j->first_index + b,
                          j->tables + b * (uint64_t)j->d * N * 4,
                          j->round_evals + b * (uint64_t)j->k * (j->d + 1) * 4,
                          j->challenges + b * (uint64_t)j->k * 4,
                          j->final_evals + b * (uint64_t)j->d * 4,
                          j->claims ? j->claims + b * 4 : NULL);
        if (s) { pthread_mutex_lock(&j->lock); j->status = s; pthread_mutex_unlock(&j->lock); }
    }
    return NULL;
}

int orc_prove_batch(uint32_t k, uint32_t d, uint32_t order, const uint8_t seed[32],
                    uint64_t first_index, uint64_t batch, const uint64_t *tables,
                    uint64_t *round_evals, uint64_t *challenges, uint64_t *final_evals,
                    uint64_t *claims, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    ensure_mu();
    batch_job j = {k, d, order, seed, first_index, batch, tables, round_evals, challenges,
                   final_evals, claims, 0, PTHREAD_MUTEX_INITIALIZER, 0};
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, batch_worker, &j);
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th);
    return j.status;
}

/* ------------------------------------------------------------------ */
/* Algorithm 1 literally: d = 1, r_i given, MSB pairing     */
/* ------------------------------------------------------------------ */
int orc_alg1(uint32_t n, const uint64_t *A_in, const uint64_t *r_in, uint64_t *pi_out) {
    if (n > 30) return ORC_EINVAL;
    ensure_mu();
    uint64_t N = (uint64_t)1 << n;
    fr *A = (fr *)malloc(sizeof(fr) * N);
    if (!A) return ORC_ENOMEM;
    for (uint64_t b = 0; b < N; ++b) memcpy(A[b].v, A_in + 4 * b, 32);
    fr one = fr_from_u64(1);
    for (uint32_t i = 1; i <= n; ++i) {                     /* line 1 */
        fr pi1 = fr_zero(), pi2 = fr_zero();
        fr ri; memcpy(ri.v, r_in + 4 * (i - 1), 32);
        uint64_t h = (uint64_t)1 << (n - i);
        for (uint64_t b = 0; b < h; ++b) {                  /* line 2 */
            pi1 = fr_add(pi1, A[b]);                        /* line 3 */
            pi2 = fr_add(pi2, A[b + h]);                    /* line 4 */
            A[b] = fr_add(fr_mul(fr_sub(one, ri), A[b]), fr_mul(ri, A[b + h]));  /* line 5 */
        }
        memcpy(pi_out + 8 * (i - 1), pi1.v, 32);
        memcpy(pi_out + 8 * (i - 1) + 4, pi2.v, 32);
    }
    free(A);
    return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* verifier                                      */
/* ------------------------------------------------------------------ */

/* g(r) from g(0..d) by Lagrange interpolation on nodes 0..d */
static fr lagrange_eval(const fr *g, uint32_t d, fr r) {
    fr acc = fr_zero();
    for (uint32_t j = 0; j <= d; ++j) {
        fr num = fr_from_u64(1), den = fr_from_u64(1);
        for (uint32_t l = 0; l <= d; ++l) {
            if (l == j) continue;
            num = fr_mul(num, fr_sub(r, fr_from_u64(l)));
            den = fr_mul(den, fr_sub(fr_from_u64(j), fr_from_u64(l)));
        }
        acc = fr_add(acc, fr_mul(g[j], fr_mul(num, fr_inv(den))));
    }
    return acc;
}

/* returns 0 on accept; otherwise 10+i (round i sum check failed), 100+i (challenge i mismatch),
 * 200 (final product check), 300 (non-canonical value), 1 (bad args) */
int orc_verify(uint32_t k, uint32_t d, uint32_t order, const uint8_t seed[32], uint64_t I,
               const uint64_t *round_evals, const uint64_t *challenges,
               const uint64_t *final_evals, const uint64_t *claim) {
    if (k > 30 || d < 1 || d > 4 || order > 1) return 1;
    ensure_mu();
    fr c; memcpy(c.v, claim, 32);
    if (!fr_is_canon(&c)) return 300;
    uint8_t state[32];
    transcript_init(state, seed, I, k, d, order);
    for (uint32_t i = 1; i <= k; ++i) {
        fr g[5];
        for (uint32_t t = 0; t <= d; ++t) {
            memcpy(g[t].v, round_evals + 4 * ((uint64_t)(i - 1) * (d + 1) + t), 32);
            if (!fr_is_canon(&g[t])) return 300;
        }
        fr s = fr_add(g[0], g[1]);
        if (!fr_eq(&s, &c)) return 10 + (int)i;
        fr r = transcript_round(state, g, d);
        fr r_given; memcpy(r_given.v, challenges + 4 * (uint64_t)(i - 1), 32);
        if (!fr_eq(&r, &r_given)) return 100 + (int)i;
        c = lagrange_eval(g, d, r);
    }
    fr prod = fr_from_u64(1);
    for (uint32_t m = 0; m < d; ++m) {
        fr f; memcpy(f.v, final_evals + 4 * m, 32);
        if (!fr_is_canon(&f)) return 300;
        prod = fr_mul(prod, f);
    }
    if (!fr_eq(&prod, &c)) return 200;
    (void)order;
    return 0;
}

/* ------------------------------------------------------------------ */
/* multilinear extension, plain definition via eq-table by doubling     */
/* point[l] is the value assigned to x_{l+1}; table index x = sum x_l 2^{l-1} */
/* ------------------------------------------------------------------ */
int orc_mle(uint32_t k, const uint64_t *table, const uint64_t *point, uint64_t *out) {
    if (k > 30) return ORC_EINVAL;
    ensure_mu();
    uint64_t N = (uint64_t)1 << k;
    fr *eq = (fr *)malloc(sizeof(fr) * N);
    if (!eq) return ORC_ENOMEM;
    eq[0] = fr_from_u64(1);
    fr one = fr_from_u64(1);
    for (uint32_t l = 0; l < k; ++l) {
        fr rho; memcpy(rho.v, point + 4 * l, 32);
        uint64_t half = (uint64_t)1 << l;
        for (uint64_t y = 0; y < half; ++y) {
            fr e = eq[y];
            eq[y + half] = fr_mul(e, rho);                 /* x_{l+1} = 1 */
            eq[y] = fr_mul(e, fr_sub(one, rho));          /* x_{l+1} = 0 */
        }
    }
    fr acc = fr_zero();
    for (uint64_t x = 0; x < N; ++x) {
        fr t; memcpy(t.v, table + 4 * x, 32);
        acc = fr_add(acc, fr_mul(t, eq[x]));
    }
    memcpy(out, acc.v, 32);
    free(eq);
    return ORC_OK;
}

/* H = sum_x prod_m T_m[x] */
int orc_hsum(uint32_t k, uint32_t d, const uint64_t *tables, uint64_t *out) {
    ensure_mu();
    uint64_t N = (uint64_t)1 << k;
    fr H = fr_zero();
    for (uint64_t x = 0; x < N; ++x) {
        fr prod; memcpy(prod.v, tables + 4 * x, 32);
        for (uint32_t m = 1; m < d; ++m) {
            fr t; memcpy(t.v, tables + 4 * ((uint64_t)m * N + x), 32);
            prod = fr_mul(prod, t);
        }
        H = fr_add(H, prod);
    }
    memcpy(out, H.v, 32);
    return ORC_OK;
}

/* element-wise field ops for pin tests: op 0 add, 1 sub, 2 mul, 3 inv, 4 reduce256 (a only) */
int orc_fr_op(int op, uint64_t n, const uint64_t *a, const uint64_t *b, uint64_t *out) {
    ensure_mu();
    for (uint64_t i = 0; i < n; ++i) {
        fr x, y, z;
        memcpy(x.v, a + 4 * i, 32);
        if (b) memcpy(y.v, b + 4 * i, 32); else y = fr_zero();
        switch (op) {
            case 0: z = fr_add(x, y); break;
            case 1: z = fr_sub(x, y); break;
            case 2: z = fr_mul(x, y); break;
            case 3: z = fr_inv(x); break;
            case 4: z = fr_from_256(x.v); break;
            default: return ORC_EINVAL;
        }
        memcpy(out + 4 * i, z.v, 32);
    }
    return ORC_OK;
}

/* expose mu for the pin test (mu = floor(2^512/p)) */
void orc_mu(uint64_t out[5]) { ensure_mu(); memcpy(out, MU, sizeof MU); }

/* ================================================================== */
/* Second field instance (reading R15): Goldilocks  */
/* p_gl = 2^64 - 2^32 + 1, elements one u64, canonical.  Same prover,   */
/* transcript framed with field id 1 (the reserved LE16 of state_0) and */
/* LE64-encoded evaluations; r_i = LE64(state_i[0..8]) mod p_gl.        */
/* Arithmetic is the plain definition: unsigned __int128 then % p.      */
/* ================================================================== */

static const uint64_t PGL = 0xffffffff00000001ULL;

static uint64_t gl_add(uint64_t a, uint64_t b) { return (uint64_t)(((u128)a + b) % PGL); }
static uint64_t gl_sub(uint64_t a, uint64_t b) { return (uint64_t)(((u128)a + PGL - b) % PGL); }
static uint64_t gl_mul(uint64_t a, uint64_t b) { return (uint64_t)(((u128)a * b) % PGL); }

static void gl_transcript_init(uint8_t state[32], const uint8_t seed[32], uint64_t I, uint32_t k, uint32_t d,
                               uint32_t order) {
    uint8_t m[64];
    memcpy(m, "BZK-SUMCHECK-V1", 15); m[15] = 0;
    memcpy(m + 16, seed, 32);
    for (int i = 0; i < 8; ++i) m[48 + i] = (uint8_t)(I >> (8 * i));
    m[56] = (uint8_t)k; m[57] = (uint8_t)(k >> 8);
    m[58] = (uint8_t)d; m[59] = (uint8_t)(d >> 8);
    m[60] = (uint8_t)order; m[61] = (uint8_t)(order >> 8);
    m[62] = 1; m[63] = 0;                                  /* field id 1 = Goldilocks */
    orc_sha256(m, 64, state);
}

static uint64_t gl_transcript_round(uint8_t state[32], const uint64_t *g, uint32_t d) {
    sha256_ctx c; sha256_init(&c);
    sha256_update(&c, state, 32);
    for (uint32_t t = 0; t <= d; ++t) {
        uint8_t b[8];
        for (int j = 0; j < 8; ++j) b[j] = (uint8_t)(g[t] >> (8 * j));
        sha256_update(&c, b, 8);
    }
    sha256_final(&c, state);
    uint64_t v = 0;
    for (int j = 0; j < 8; ++j) v |= (uint64_t)state[j] << (8 * j);
    return v % PGL;
}

/* One Goldilocks proof: tables [d][2^k] u64; round_evals [k][d+1]; challenges [k]; final [d];
 * claim [1].  given_r (may be NULL): paper-literal mode, challenges are inputs. */
int orc_gl_prove(uint32_t k, uint32_t d, uint32_t order, const uint8_t seed[32], uint64_t I,
                 const uint64_t *tables, const uint64_t *given_r, uint64_t *round_evals, uint64_t *challenges,
                 uint64_t *final_evals, uint64_t *claim) {
    if (k > 30 || d < 1 || d > 4 || order > 1) return ORC_EINVAL;
    const uint64_t N = (uint64_t)1 << k;
    uint64_t *T = (uint64_t *)malloc(sizeof(uint64_t) * N * d);
    if (!T) return ORC_ENOMEM;
    for (uint64_t x = 0; x < N * d; ++x) {
        if (tables[x] >= PGL) { free(T); return ORC_ENONCANON; }
        T[x] = tables[x];
    }
    uint64_t H = 0;
    for (uint64_t x = 0; x < N; ++x) {
        uint64_t prod = T[x];
        for (uint32_t m = 1; m < d; ++m) prod = gl_mul(prod, T[m * N + x]);
        H = gl_add(H, prod);
    }
    uint8_t state[32];
    gl_transcript_init(state, seed, I, k, d, order);
    uint64_t size = N, g[5];
    for (uint32_t i = 1; i <= k; ++i) {
        uint64_t h = size / 2;
        for (uint32_t t = 0; t <= d; ++t) {
            uint64_t acc = 0;
            for (uint64_t j = 0; j < h; ++j) {
                uint64_t prod = 1;
                for (uint32_t m = 0; m < d; ++m) {
                    const uint64_t *Tm = T + (uint64_t)m * N;
                    uint64_t a = order == 0 ? Tm[2 * j] : Tm[j];
                    uint64_t b = order == 0 ? Tm[2 * j + 1] : Tm[j + h];
                    prod = gl_mul(prod, gl_add(a, gl_mul(t, gl_sub(b, a))));
                }
                acc = gl_add(acc, prod);
            }
            g[t] = acc;
        }
        uint64_t r;
        if (given_r) {
            r = given_r[i - 1];
            if (r >= PGL) { free(T); return ORC_ENONCANON; }
        } else {
            r = gl_transcript_round(state, g, d);
        }
        for (uint32_t t = 0; t <= d; ++t) round_evals[(uint64_t)(i - 1) * (d + 1) + t] = g[t];
        challenges[i - 1] = r;
        for (uint32_t m = 0; m < d; ++m) {
            uint64_t *Tm = T + (uint64_t)m * N;
            for (uint64_t j = 0; j < h; ++j) {
                uint64_t a = order == 0 ? Tm[2 * j] : Tm[j];
                uint64_t b = order == 0 ? Tm[2 * j + 1] : Tm[j + h];
                Tm[j] = gl_add(a, gl_mul(r, gl_sub(b, a)));
            }
        }
        size = h;
    }
    for (uint32_t m = 0; m < d; ++m) final_evals[m] = T[(uint64_t)m * N];
    if (claim) claim[0] = H;
    free(T);
    return ORC_OK;
}

/* element-wise Goldilocks ops for pins: op 0 add, 1 sub, 2 mul */
int orc_gl_op(int op, uint64_t n, const uint64_t *a, const uint64_t *b, uint64_t *out) {
    for (uint64_t i = 0; i < n; ++i) {
        switch (op) {
            case 0: out[i] = gl_add(a[i] % PGL, b[i] % PGL); break;
            case 1: out[i] = gl_sub(a[i] % PGL, b[i] % PGL); break;
            case 2: out[i] = gl_mul(a[i] % PGL, b[i] % PGL); break;
            default: return ORC_EINVAL;
        }
    }
    return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* Merkle trees (readings R17-R19)       */
/*   P:91-97 Sec. 2.2 Fig. 2: "divides input data into multiple blocks  */
/*   and then hashes each block to create the leaf node ... iteratively */
/*   combines pairs of these hash values ... until only one hash value  */
/*   remains at the top, known as the Merkle root".                     */
/*   P:137 Sec. 3.1: N 512-bit blocks, log N rounds; 2N hashes.  */
/* Hash H of a 512-bit block (reading R18):                             */
/*   mode 0 (paper-literal, "produces a fixed-size 256-bit hash    */
/*     value from a 512-bit block"): one SHA-256 compression of the     */
/*     block from the FIPS 180-4 initial value, digest = the 8 state    */
/*     words big-endian;                                                */
/*   mode 1: the full FIPS 180-4 SHA-256 of the 64-byte message.        */
/* Nodes, level-major (reading R19): level 0 = N leaf digests           */
/* H(block_x); level l+1 [j] = H(level_l[2j] || level_l[2j+1]); the     */
/* root is level n [0]; 2N-1 digests per tree.                          */
/* ------------------------------------------------------------------ */

/* one compression from an arbitrary state (exposed for the pins)     */
void orc_sha256_compress(const uint32_t h_in[8], const uint8_t blk[64], uint32_t h_out[8]) {
    uint32_t h[8];
    memcpy(h, h_in, sizeof h);
    sha256_block(h, blk);
    memcpy(h_out, h, sizeof h);
}

static void merkle_hash(const uint8_t blk[64], int mode, uint8_t out[32]) {
    if (mode == 1) { orc_sha256(blk, 64, out); return; }
    static const uint32_t IV[8] = {0x6a09e667, 0xbb67ae85, 0x3c6ef372, 0xa54ff53a,
                                   0x510e527f, 0x9b05688c, 0x1f83d9ab, 0x5be0cd19};
    uint32_t h[8];
    memcpy(h, IV, sizeof h);
    sha256_block(h, blk);
    for (int i = 0; i < 8; ++i) {
        out[4 * i] = (uint8_t)(h[i] >> 24); out[4 * i + 1] = (uint8_t)(h[i] >> 16);
        out[4 * i + 2] = (uint8_t)(h[i] >> 8); out[4 * i + 3] = (uint8_t)h[i];
    }
}

/* One tree of N = 2^n blocks (64 bytes each).  nodes: (2N-1) x 32 bytes, level-major, or NULL.
 * root: 32 bytes.  Level by level exactly as P:97 describes it. */
int orc_merkle(uint32_t n, int mode, const uint8_t *blocks, uint8_t *nodes, uint8_t root[32]) {
    if (n > 24 || (mode != 0 && mode != 1)) return 1;
    const uint64_t N = (uint64_t)1 << n;
    uint8_t *lv = (uint8_t *)malloc((size_t)(2 * N - 1) * 32);
    if (!lv) return 2;
    /* level 0: leaf digests */
    for (uint64_t x = 0; x < N; ++x) merkle_hash(blocks + 64 * x, mode, lv + 32 * x);
    /* level l+1 from level l: the concatenation of two adjacent digests is a 512-bit block */
    uint64_t off = 0, cnt = N;
    while (cnt > 1) {
        uint8_t *cur = lv + 32 * off, *nxt = lv + 32 * (off + cnt);
        for (uint64_t j = 0; j < cnt / 2; ++j) {
            uint8_t blk[64];
            memcpy(blk, cur + 64 * j, 32);
            memcpy(blk + 32, cur + 64 * j + 32, 32);
            merkle_hash(blk, mode, nxt + 32 * j);
        }
        off += cnt;
        cnt /= 2;
    }
    memcpy(root, lv + 32 * off, 32);
    if (nodes) memcpy(nodes, lv, (size_t)(2 * N - 1) * 32);
    free(lv);
    return 0;
}

/* Authentication path of block x (siblings from the leaf level up, n x 32 bytes), read from a
 * level-major node array, and its check: recompute the root from the block and the path. */
int orc_merkle_path(uint32_t n, const uint8_t *nodes, uint64_t x, uint8_t *path) {
    uint64_t off = 0, cnt = (uint64_t)1 << n;
    for (uint32_t l = 0; l < n; ++l) {
        memcpy(path + 32 * l, nodes + 32 * (off + (x ^ 1)), 32);
        off += cnt; cnt /= 2; x /= 2;
    }
    return 0;
}

int orc_merkle_verify_path(uint32_t n, int mode, const uint8_t blk[64], uint64_t x, const uint8_t *path,
                           const uint8_t root[32]) {
    uint8_t cur[32], buf[64];
    merkle_hash(blk, mode, cur);
    for (uint32_t l = 0; l < n; ++l) {
        if (x & 1) { memcpy(buf, path + 32 * l, 32); memcpy(buf + 32, cur, 32); }
        else       { memcpy(buf, cur, 32); memcpy(buf + 32, path + 32 * l, 32); }
        merkle_hash(buf, mode, cur);
        x /= 2;
    }
    return memcmp(cur, root, 32) == 0;
}

typedef struct {
    uint32_t n; int mode; uint64_t batch; const uint8_t *blocks; uint8_t *nodes, *roots;
    uint64_t next; pthread_mutex_t lock; int status;
} merkle_job;

static void *merkle_worker(void *arg) {
    merkle_job *j = (merkle_job *)arg;
    const uint64_t N = (uint64_t)1 << j->n;
    for (;;) {
        pthread_mutex_lock(&j->lock);
        uint64_t b = j->next++;
        pthread_mutex_unlock(&j->lock);
        if (b >= j->batch) break;
        int s = orc_merkle(j->n, j->mode, j->blocks + b * N * 64,
                           j->nodes ? j->nodes + b * (2 * N - 1) * 32 : NULL, j->roots + b * 32);
        if (s) { pthread_mutex_lock(&j->lock); j->status = s; pthread_mutex_unlock(&j->lock); }
    }
    return NULL;
}

int orc_merkle_batch(uint32_t n, int mode, uint64_t batch, const uint8_t *blocks, uint8_t *nodes,
                     uint8_t *roots, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    merkle_job j = {n, mode, batch, blocks, nodes, roots, 0, PTHREAD_MUTEX_INITIALIZER, 0};
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, merkle_worker, &j);
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th);
    return j.status;
}

/* ------------------------------------------------------------------ */
/* Linear-time (Spielman-style) encoder (readings   */
/* R21-R24).  P:113-117 Sec. 2.4, Fig. 3: each stage         */
/* multiplies its input by the first bipartite graph's sparse matrix,    */
/* encodes the result recursively ("forwarded to the subsequent stage"), */
/* multiplies the returned vector by the second graph's matrix; "the     */
/* result, combined with the input vector and the vector returned from   */
/* the subsequent stage, forms the output of this stage".  Rows = right  */
/* vertices, columns = left vertices.  Written recursively,      */
/* exactly in that order (the GPU path is iterative).         */
/*   Enc_l(x), |x| = n_l:  l == L: x || G0 x  (base code)                */
/*                         else    y = A_l x; z = Enc_{l+1}(y);          */
/*                                 w = B_l z; return x || z || w         */
/* ------------------------------------------------------------------ */

typedef struct { uint32_t rows, cols; const uint32_t *row_ptr, *col; const uint64_t *val; } orc_csr;

/* y[r] = sum over the row's edges (r, j) of val * x[j]  (plain: fr_mul, fr_add per edge) */
static void csr_apply(const orc_csr *M, const fr *x, fr *y) {
    for (uint32_t r = 0; r < M->rows; ++r) {
        fr acc = fr_zero();
        for (uint32_t e = M->row_ptr[r]; e < M->row_ptr[r + 1]; ++e) {
            fr w; memcpy(w.v, M->val + 4 * (uint64_t)e, 32);
            acc = fr_add(acc, fr_mul(w, x[M->col[e]]));
        }
        y[r] = acc;
    }
}

static int enc_rec(uint32_t l, uint32_t levels, const orc_csr *A, const orc_csr *B, const orc_csr *G0,
                   const fr *x, uint64_t n, fr *out) {
    memcpy(out, x, n * sizeof(fr));                    /* the input vector is part of the output */
    if (l == levels) {                                 /* base code: x || G0 x */
        if (G0->cols != n || G0->rows != n) return 1;
        csr_apply(G0, x, out + n);
        return 0;
    }
    if (A[l].cols != n || A[l].rows != n / 4 || B[l].cols != n / 2 || B[l].rows != n / 2) return 1;
    fr *y = (fr *)malloc((n / 4) * sizeof(fr));
    if (!y) return 2;
    csr_apply(&A[l], x, y);                            /* first vector-matrix multiplication */
    int s = enc_rec(l + 1, levels, A, B, G0, y, n / 4, out + n);   /* z = Enc(y), length n/2 */
    free(y);
    if (s) return s;
    csr_apply(&B[l], out + n, out + n + n / 2);        /* second: w = B z */
    return 0;
}

/* msg: n = 2^log_n canonical elements [n][4]; out: codeword [2n][4] = x || z || w */
int orc_encode(uint32_t log_n, uint32_t levels, const orc_csr *A, const orc_csr *B, const orc_csr *G0,
               const uint64_t *msg, uint64_t *out) {
    ensure_mu();
    const uint64_t n = (uint64_t)1 << log_n;
    for (uint64_t i = 0; i < n; ++i) {
        fr t; memcpy(t.v, msg + 4 * i, 32);
        if (!fr_is_canon(&t)) return 3;
    }
    return enc_rec(0, levels, A, B, G0, (const fr *)msg, n, (fr *)out);
}

typedef struct {
    uint32_t log_n, levels; const orc_csr *A, *B, *G0; uint64_t batch; const uint64_t *msgs; uint64_t *out;
    uint64_t next; pthread_mutex_t lock; int status;
} enc_job;

static void *enc_worker(void *arg) {
    enc_job *j = (enc_job *)arg;
    const uint64_t n = (uint64_t)1 << j->log_n;
    for (;;) {
        pthread_mutex_lock(&j->lock);
        uint64_t b = j->next++;
        pthread_mutex_unlock(&j->lock);
        if (b >= j->batch) break;
        int s = orc_encode(j->log_n, j->levels, j->A, j->B, j->G0, j->msgs + b * n * 4, j->out + b * 2 * n * 4);
        if (s) { pthread_mutex_lock(&j->lock); j->status = s; pthread_mutex_unlock(&j->lock); }
    }
    return NULL;
}

int orc_encode_batch(uint32_t log_n, uint32_t levels, const orc_csr *A, const orc_csr *B, const orc_csr *G0,
                     uint64_t batch, const uint64_t *msgs, uint64_t *out, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    ensure_mu();
    enc_job j = {log_n, levels, A, B, G0, batch, msgs, out, 0, PTHREAD_MUTEX_INITIALIZER, 0};
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, enc_worker, &j);
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th);
    return j.status;
}
