"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no field operations): it
only turns a counter into 64-bit words.  The one place a modulus appears is the
range of the generated values -- they must be canonical field elements, so a
value drawn from [0, 2^254) that lands in [p, 2^254) is moved down by p once
(a comparison and a subtraction on raw words, SURVEY.md 8(d) "mask to 254 bits;
if >= p, subtract p once").  The CUDA side implements the same counter-based
generator in ``csrc/gen.cuh`` (``bzk_generate``); the two are checked
word-for-word by ``tests/test_gpu_parity.py::test_generator_matches_host_twin``.

Recipe:
    ctr(I, m, x, w) = (I << 36) | (m << 32) | (x << 2) | w          I < 2^28, m < 16, x < 2^30, w < 4
    word            = splitmix64_mix(data_seed + (ctr + 1) * 0x9E3779B97F4A7C15)
    uniform  : limbs w = 0..3 are the words, limb 3 masked to 62 bits (value < 2^254), then one
               conditional subtraction of p -> uniform-ish over the WHOLE field [0, p)
    smallint : limb 0 = word(w=0) & 0xff, limbs 1..3 = 0 (non-negative 8-bit activations, VML)
    vml      : table m = 0 smallint, tables m >= 1 uniform
    adversarial : the operands where lazy reduction bounds are tightest.  Each table (I, m) draws a
               mode from  word'(I, m) mod 5  (word' = splitmix64 with data_seed ^ ADV_TABLE_SALT at
               ctr = I << 36 | m << 32):
                 0 near-top   p - 1 - (word(w=0) & 0xffff)      in [p - 2^16, p)
                 1 all p - 1
                 2 alternating 0 (x even) / p - 1 (x odd)
                 3 high band  [2^253, 2^253 + 2^252)  (limb 3 = (word(w=3) & (2^60 - 1)) | 2^61)
                 4 per-element mix: word''(I, m, x) mod 5 (salt ADV_ELEM_SALT) picks near-top,
                   p - 1, 0, high band or uniform for each element
I is the GLOBAL proof index, so a proof's tables do not depend on the batch it
is generated in, the wave it runs in or the GPU it is sharded to.
"""
from __future__ import annotations

import numpy as np

DATA_SEED = 0x42415443485A4B31          # "BATCHZK1"
DEFAULT_SEED = bytes(range(32))          # transcript seed 0x00..0x1f (stands in for a Merkle root)

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
M1 = np.uint64(0xBF58476D1CE4E5B9)
M2 = np.uint64(0x94D049BB133111EB)
MASK61 = np.uint64((1 << 61) - 1)

DIST_UNIFORM = 0
DIST_SMALLINT = 1
DIST_VML = 2
DIST_GL = 3          # Goldilocks (NEXT-2): ONE word per element, one conditional subtraction of p_gl
DIST_ADV = 4         # BN254 adversarial (top of the field, p - 1, 0 / p - 1, [2^253, ...)), see above
DIST_GL_ADV = 5      # Goldilocks adversarial: the same five modes over p_gl, high band [2^63, p_gl)
DISTS = {"uniform": DIST_UNIFORM, "smallint": DIST_SMALLINT, "vml": DIST_VML, "gl": DIST_GL,
         "adversarial": DIST_ADV, "gl_adversarial": DIST_GL_ADV}
MASK62 = np.uint64((1 << 62) - 1)
MASK60 = np.uint64((1 << 60) - 1)
BIT61 = np.uint64(1 << 61)

# range bounds of the generated values (the field moduli, as raw 64-bit words; no arithmetic mod p)
P_BN254 = [0x43E1F593F0000001, 0x2833E84879B97091, 0xB85045B68181585D, 0x30644E72E131A029]
P_GL = 0xFFFFFFFF00000001
ADV_TABLE_SALT = 0x5441424C45414456     # "TABLEADV"
ADV_ELEM_SALT = 0x454C454D41445653      # "ELEMADVS"


def splitmix64(ctr: np.ndarray, data_seed: int = DATA_SEED) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = np.uint64(data_seed) + (ctr.astype(np.uint64) + np.uint64(1)) * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
        return z ^ (z >> np.uint64(31))


def _geq_p(words: np.ndarray) -> np.ndarray:
    """words [..., 4] (LE u64) >= p_bn254, lexicographically from the top limb."""
    ge = np.ones(words.shape[:-1], dtype=bool)          # equal so far -> >= holds on full equality
    for i in range(4):                                  # from the lowest limb up: top limbs decide last
        pi = np.uint64(P_BN254[i])
        ge = (words[..., i] > pi) | ((words[..., i] == pi) & ge)
    return ge


def _sub_p(words: np.ndarray) -> np.ndarray:
    """words - p_bn254 (words >= p), 4-limb subtraction with borrow."""
    out = np.empty_like(words)
    borrow = np.zeros(words.shape[:-1], dtype=np.uint64)
    with np.errstate(over="ignore"):
        for i in range(4):
            pi = np.uint64(P_BN254[i])
            out[..., i] = words[..., i] - pi - borrow
            borrow = ((words[..., i] < pi) | ((words[..., i] == pi) & (borrow == 1))).astype(np.uint64)
    return out


def _canonical_254(words: np.ndarray) -> np.ndarray:
    """mask limb 3 to 62 bits (value < 2^254 < 2p), then subtract p once where value >= p"""
    words = words.copy()
    words[..., 3] &= MASK62
    ge = _geq_p(words)
    if ge.any():
        words[ge] = _sub_p(words[ge])
    return words


def _pm1(shape) -> np.ndarray:
    out = np.empty(tuple(shape) + (4,), dtype=np.uint64)
    out[...] = np.array(P_BN254, dtype=np.uint64)
    out[..., 0] -= np.uint64(1)
    return out


def _adv_modes(I: int, m: int, x: np.ndarray, data_seed: int):
    """(table mode, per-element mode array): table mode 0..3 applies to every element; table mode 4
    gives each element its own mode 0..4 (0 near-top, 1 p - 1, 2 ZERO, 3 high band, 4 uniform)."""
    base = (np.uint64(I) << np.uint64(36)) | (np.uint64(m) << np.uint64(32))
    tmode = int(splitmix64(np.array([base], dtype=np.uint64), data_seed ^ ADV_TABLE_SALT)[0] % np.uint64(5))
    if tmode < 4:
        return tmode, np.full(x.shape, tmode, dtype=np.int64)
    return tmode, (splitmix64(base | (x << np.uint64(2)), data_seed ^ ADV_ELEM_SALT) % np.uint64(5)).astype(np.int64)


def _adversarial(I: int, m: int, x: np.ndarray, words: np.ndarray, data_seed: int) -> np.ndarray:
    """BN254 adversarial table (DIST_ADV), modes as in the module docstring."""
    tmode, mode = _adv_modes(I, m, x, data_seed)
    out = _canonical_254(words)                                  # element mode 4: uniform
    near = _pm1(x.shape)
    near[..., 0] -= words[..., 0] & np.uint64(0xFFFF)            # p - 1 - s, s < 2^16 (limb 0 of p - 1 >= 2^16)
    out[mode == 0] = near[mode == 0]
    out[mode == 1] = _pm1(x.shape)[mode == 1]
    two = _pm1(x.shape)
    two[(x & np.uint64(1)) == 0] = 0                             # table mode 2: 0 / p - 1 alternating
    if tmode == 4:
        two[:] = 0                                               # element mode 2: zero
    out[mode == 2] = two[mode == 2]
    high = words.copy()
    high[..., 3] = (high[..., 3] & MASK60) | BIT61               # [2^253, 2^253 + 2^252)
    out[mode == 3] = high[mode == 3]
    return out


def gen_tables_gl(batch: int, d: int, k: int, first_index: int = 0, data_seed: int = DATA_SEED,
                  dist: str | int = "gl") -> np.ndarray:
    """Goldilocks tables, uint64 [B][d][2^k]: word(I, m, x, w=0), minus p_gl once if >= p_gl
    ("gl"), or the adversarial modes over p_gl ("gl_adversarial": high band [2^63, 2^63 + 2^62))."""
    dist = DISTS[dist] if isinstance(dist, str) else int(dist)
    N = 1 << k
    out = np.empty((batch, d, N), dtype=np.uint64)
    x = np.arange(N, dtype=np.uint64)
    pgl = np.uint64(P_GL)
    for bi in range(batch):
        I = first_index + bi
        for m in range(d):
            ctr = (np.uint64(I) << np.uint64(36)) | (np.uint64(m) << np.uint64(32)) | (x << np.uint64(2))
            w = splitmix64(ctr, data_seed)
            uni = np.where(w >= pgl, w - pgl, w)
            if dist != DIST_GL_ADV:
                out[bi, m] = uni
                continue
            tmode, mode = _adv_modes(I, m, x, data_seed)
            v = uni.copy()
            v[mode == 0] = (pgl - np.uint64(1) - (w & np.uint64(0xFFFF)))[mode == 0]
            v[mode == 1] = pgl - np.uint64(1)
            two = np.where((x & np.uint64(1)) == 0, np.uint64(0), pgl - np.uint64(1))
            if tmode == 4:
                two[:] = 0
            v[mode == 2] = two[mode == 2]
            v[mode == 3] = ((w & np.uint64((1 << 62) - 1)) | np.uint64(1 << 63))[mode == 3]
            out[bi, m] = v
    return out


def gen_tables(batch: int, d: int, k: int, first_index: int = 0, dist: str | int = "uniform",
               data_seed: int = DATA_SEED, indices=None) -> np.ndarray:
    """uint64 [B][d][2^k][4] tables for global proof indices first_index.. (or ``indices``)."""
    dist = DISTS[dist] if isinstance(dist, str) else int(dist)
    assert 0 <= k <= 30 and 1 <= d <= 15 and dist in (DIST_UNIFORM, DIST_SMALLINT, DIST_VML, DIST_ADV)
    idx = np.arange(first_index, first_index + batch, dtype=np.uint64) if indices is None \
        else np.asarray(indices, dtype=np.uint64)
    N = 1 << k
    out = np.empty((len(idx), d, N, 4), dtype=np.uint64)
    x = np.arange(N, dtype=np.uint64)
    w = np.arange(4, dtype=np.uint64)
    for bi, I in enumerate(idx):
        for m in range(d):
            base = (np.uint64(I) << np.uint64(36)) | (np.uint64(m) << np.uint64(32))
            ctr = base | (x[:, None] << np.uint64(2)) | w[None, :]
            words = splitmix64(ctr, data_seed)
            small = dist == DIST_SMALLINT or (dist == DIST_VML and m == 0)
            if small:
                out[bi, m, :, 0] = words[:, 0] & np.uint64(0xFF)
                out[bi, m, :, 1:] = 0
            elif dist == DIST_ADV:
                out[bi, m] = _adversarial(int(I), m, x, words, data_seed)
            else:
                out[bi, m] = _canonical_254(words)
    return out


# ---------------------------------------------------------------- Merkle blocks (NEXT-3)
# ctr(I, x, w) = (I << 36) | (x << 3) | w   (I < 2^28, x < 2^33, w < 8); a block is the 8 words
# LE64-serialised, 64 bytes.  Device twin: gen.cuh k_generate_blocks (bzk_generate_blocks).
MERKLE_DATA_SEED = 0x42415443485A4B4D   # "BATCHZKM"


def gen_blocks(batch: int, n: int, first_index: int = 0, data_seed: int = MERKLE_DATA_SEED) -> np.ndarray:
    """uint8 [B][2^n][64] Merkle input blocks for global tree indices first_index.."""
    N = 1 << n
    out = np.empty((batch, N, 8), dtype=np.uint64)
    x = np.arange(N, dtype=np.uint64)
    w = np.arange(8, dtype=np.uint64)
    for bi in range(batch):
        I = np.uint64(first_index + bi)
        ctr = (I << np.uint64(36)) | (x[:, None] << np.uint64(3)) | w[None, :]
        out[bi] = splitmix64(ctr, data_seed)
    return out.astype("<u8").view(np.uint8).reshape(batch, N, 64)


# ---------------------------------------------------------------- linear-time encoder graphs (NEXT-4)
# The Spielman-style code's random bipartite graphs are INPUTS of the method (the random draws are
# passed in, readings R21-R24).  Counter: ctr = ((((l << 2 | mat) << 24 | j) << 8 | t) << 3) | w
# for level l < 16, matrix mat (0 = A_l, 1 = B_l, 2 = base G0), left vertex j < 2^24, edge t < 256,
# word w (0..3 weight limbs, 4 = row pick).  Left-regular graphs: every left vertex (input) picks
# `deg` distinct right vertices (rows); a duplicate pick moves to the next row (mod rows).
# Weights: uniform < 2^253, limb 0 | 1 (nonzero).  Rows = right vertices.
ENC_DATA_SEED = 0x42415443485A4B45     # "BATCHZKE"
ENC_C, ENC_D = 10, 20                  # left degrees of A_l and B_l (reading R22)


def enc_levels(log_n: int, log_n0: int) -> int:
    """Recursion depth L: level l encodes n_l = n / 4^l elements; the base code takes n_L <= n0."""
    L = 0
    while log_n - 2 * L > log_n0:
        L += 1
    return L


def _enc_ctr(l, mat, j, t, w):
    j = np.asarray(j, dtype=np.uint64)
    t = np.asarray(t, dtype=np.uint64)
    return (((((np.uint64(l) << np.uint64(2) | np.uint64(mat)) << np.uint64(24) | j) << np.uint64(8) | t)
             << np.uint64(3)) | np.uint64(w))


def _left_regular_csr(l, mat, cols, rows, deg, seed):
    j = np.arange(cols, dtype=np.uint64)[:, None]
    t = np.arange(deg, dtype=np.uint64)[None, :]
    r = (splitmix64(_enc_ctr(l, mat, j, t, 4), seed) % np.uint64(rows)).astype(np.int64)
    for q in range(1, deg):
        dup = (r[:, :q] == r[:, q:q + 1]).any(axis=1)
        while dup.any():
            r[dup, q] = (r[dup, q] + 1) % rows
            dup = (r[:, :q] == r[:, q:q + 1]).any(axis=1)
    w = np.stack([splitmix64(_enc_ctr(l, mat, j, t, k), seed) for k in range(4)], axis=-1)
    w[..., 3] &= MASK61
    w[..., 0] |= np.uint64(1)
    rr = r.reshape(-1)
    cc = np.repeat(np.arange(cols, dtype=np.int64), deg)
    order = np.lexsort((cc, rr))
    row_ptr = np.zeros(rows + 1, dtype=np.uint32)
    np.cumsum(np.bincount(rr, minlength=rows), out=row_ptr[1:])
    return {"rows": rows, "cols": cols, "row_ptr": row_ptr, "col": cc[order].astype(np.uint32),
            "val": np.ascontiguousarray(w.reshape(-1, 4)[order])}


def _dense_csr(l, m, seed):
    i = np.arange(m, dtype=np.uint64)[:, None]
    jj = np.arange(m, dtype=np.uint64)[None, :]
    idx = i * np.uint64(m) + jj
    w = np.stack([splitmix64(_enc_ctr(l, 2, idx, 0, k), seed) for k in range(4)], axis=-1)
    w[..., 3] &= MASK61
    w[..., 0] |= np.uint64(1)
    return {"rows": m, "cols": m, "row_ptr": (np.arange(m + 1, dtype=np.uint32) * np.uint32(m)),
            "col": np.tile(np.arange(m, dtype=np.uint32), m), "val": np.ascontiguousarray(w.reshape(-1, 4))}


def gen_code(log_n: int, log_n0: int = 6, c: int = ENC_C, d: int = ENC_D, seed: int = ENC_DATA_SEED) -> dict:
    """Graphs of the code for messages of n = 2^log_n elements: per level l < L, A_l (n_l/4 rows x n_l
    cols, left degree c) and B_l (n_l/2 x n_l/2, left degree d); the base G0 (m x m dense, m = n_L)."""
    assert 6 <= log_n0 and log_n <= 24
    L = enc_levels(log_n, log_n0)
    A, B = [], []
    for l in range(L):
        nl = 1 << (log_n - 2 * l)
        A.append(_left_regular_csr(l, 0, nl, nl // 4, c, seed))
        B.append(_left_regular_csr(l, 1, nl // 2, nl // 2, d, seed))
    m = 1 << (log_n - 2 * L)
    return {"log_n": log_n, "log_n0": log_n0, "levels": L, "A": A, "B": B, "G0": _dense_csr(L, m, seed), "m": m}
