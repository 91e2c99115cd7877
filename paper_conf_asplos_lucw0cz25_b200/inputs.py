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
