"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no field operations, no
modulus): it only turns a counter into 64-bit words.  The CUDA side implements
the same counter-based generator in ``csrc/gen.cu`` (``bzk_generate``); the two
are checked word-for-word by ``tests/test_gpu_generator.py``.

Recipe:
    ctr(I, m, x, w) = (I << 36) | (m << 32) | (x << 2) | w          I < 2^28, m < 16, x < 2^30, w < 4
    word            = splitmix64_mix(data_seed + (ctr + 1) * 0x9E3779B97F4A7C15)
    uniform  : limbs w = 0..3 are the words, limb 3 masked to 61 bits -> value < 2^253 < p
    smallint : limb 0 = word(w=0) & 0xff, limbs 1..3 = 0 (non-negative 8-bit activations, VML)
    vml      : table m = 0 smallint, tables m >= 1 uniform
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
DIST_GL = 3          # Goldilocks (NEXT-2): ONE word per element, masked to 63 bits -> < 2^63 < p_gl
DISTS = {"uniform": DIST_UNIFORM, "smallint": DIST_SMALLINT, "vml": DIST_VML, "gl": DIST_GL}
MASK63 = np.uint64((1 << 63) - 1)


def splitmix64(ctr: np.ndarray, data_seed: int = DATA_SEED) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = np.uint64(data_seed) + (ctr.astype(np.uint64) + np.uint64(1)) * GOLDEN
        z = (z ^ (z >> np.uint64(30))) * M1
        z = (z ^ (z >> np.uint64(27))) * M2
        return z ^ (z >> np.uint64(31))


def gen_tables_gl(batch: int, d: int, k: int, first_index: int = 0, data_seed: int = DATA_SEED) -> np.ndarray:
    """Goldilocks tables, uint64 [B][d][2^k]: word(I, m, x, w=0) & (2^63 - 1)."""
    N = 1 << k
    out = np.empty((batch, d, N), dtype=np.uint64)
    x = np.arange(N, dtype=np.uint64)
    for bi in range(batch):
        I = np.uint64(first_index + bi)
        for m in range(d):
            ctr = (I << np.uint64(36)) | (np.uint64(m) << np.uint64(32)) | (x << np.uint64(2))
            out[bi, m] = splitmix64(ctr, data_seed) & MASK63
    return out


def gen_tables(batch: int, d: int, k: int, first_index: int = 0, dist: str | int = "uniform",
               data_seed: int = DATA_SEED, indices=None) -> np.ndarray:
    """uint64 [B][d][2^k][4] tables for global proof indices first_index.. (or ``indices``)."""
    dist = DISTS[dist] if isinstance(dist, str) else int(dist)
    assert 0 <= k <= 30 and 1 <= d <= 15
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
            else:
                words[:, 3] &= MASK61
                out[bi, m] = words
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
