"""Python cross-oracle for batched Merkle trees -- tiny trees only.

TEST INFRASTRUCTURE ONLY -- never imported by the product path.

Independent of ``oracle/oracle.c`` and of the CUDA path:

* ``sha256_compress`` -- the SHA-256 compression function written from FIPS 180-4
  Sec. 6.2.2, with its constants *derived* from their definition (Sec. 4.2.2 / 5.3.3:
  the first 32 bits of the fractional parts of the cube roots of the first 64 primes and
  of the square roots of the first 8 primes), by exact integer roots -- no typed table.
* ``merkle_root_recursive`` -- the root from the recursive definition
  root(T) = H(root(left half) || root(right half)), root(single block) = H(block)
  (Sec. 2.2 Fig. 2), a different formulation from the oracle's level-by-level loop.
* ``merkle_levels`` -- all levels, level-major (reading R19).

H (reading R18): mode 0 = one compression of the 512-bit block from the IV ("a fixed-size
256-bit hash value from a 512-bit block"); mode 1 = ``hashlib.sha256`` of the 64-byte message.
"""
from __future__ import annotations

import hashlib
import struct

MASK = 0xFFFFFFFF


def _primes(n: int) -> list[int]:
    out, c = [], 2
    while len(out) < n:
        if all(c % p for p in out if p * p <= c):
            out.append(c)
        c += 1
    return out


def _iroot(x: int, e: int) -> int:
    """floor(x^(1/e)) for integers by Newton's method."""
    if x < 2:
        return x
    r = 1 << ((x.bit_length() + e - 1) // e)
    while True:
        s = ((e - 1) * r + x // r ** (e - 1)) // e
        if s >= r:
            return r
        r = s


# FIPS 180-4 Sec. 4.2.2: K_t = first 32 bits of frac(cbrt(prime_t)); Sec. 5.3.3: H0_i from sqrt.
K = [_iroot(p << 96, 3) & MASK for p in _primes(64)]
IV = [_iroot(p << 64, 2) & MASK for p in _primes(8)]


def _rotr(x: int, n: int) -> int:
    return ((x >> n) | (x << (32 - n))) & MASK


def sha256_compress(state: list[int], block: bytes) -> list[int]:
    """FIPS 180-4 Sec. 6.2.2 steps 1-4 for one 512-bit block."""
    assert len(block) == 64 and len(state) == 8
    W = list(struct.unpack(">16I", block))
    for t in range(16, 64):
        s0 = _rotr(W[t - 15], 7) ^ _rotr(W[t - 15], 18) ^ (W[t - 15] >> 3)
        s1 = _rotr(W[t - 2], 17) ^ _rotr(W[t - 2], 19) ^ (W[t - 2] >> 10)
        W.append((s1 + W[t - 7] + s0 + W[t - 16]) & MASK)
    a, b, c, d, e, f, g, h = state
    for t in range(64):
        T1 = (h + (_rotr(e, 6) ^ _rotr(e, 11) ^ _rotr(e, 25)) + ((e & f) ^ (~e & g)) + K[t] + W[t]) & MASK
        T2 = ((_rotr(a, 2) ^ _rotr(a, 13) ^ _rotr(a, 22)) + ((a & b) ^ (a & c) ^ (b & c))) & MASK
        h, g, f, e, d, c, b, a = g, f, e, (d + T1) & MASK, c, b, a, (T1 + T2) & MASK
    return [(x + y) & MASK for x, y in zip(state, [a, b, c, d, e, f, g, h])]


def sha256_pad(msg: bytes) -> bytes:
    """FIPS 180-4 Sec. 5.1.1 padding."""
    L = len(msg) * 8
    m = msg + b"\x80" + b"\x00" * ((55 - len(msg)) % 64) + L.to_bytes(8, "big")
    assert len(m) % 64 == 0
    return m


def sha256_from_compress(msg: bytes) -> bytes:
    """Full SHA-256 = padding + iterated compression (used to pin ``sha256_compress`` to hashlib)."""
    h = list(IV)
    m = sha256_pad(msg)
    for i in range(0, len(m), 64):
        h = sha256_compress(h, m[i:i + 64])
    return struct.pack(">8I", *h)


def H(block: bytes, mode: int) -> bytes:
    assert len(block) == 64
    if mode == 1:
        return hashlib.sha256(block).digest()
    return struct.pack(">8I", *sha256_compress(list(IV), block))


def merkle_root_recursive(blocks: list[bytes], mode: int) -> bytes:
    if len(blocks) == 1:
        return H(blocks[0], mode)
    half = len(blocks) // 2
    return H(merkle_root_recursive(blocks[:half], mode) + merkle_root_recursive(blocks[half:], mode), mode)


def merkle_levels(blocks: list[bytes], mode: int) -> list[list[bytes]]:
    lv = [[H(b, mode) for b in blocks]]
    while len(lv[-1]) > 1:
        c = lv[-1]
        lv.append([H(c[2 * j] + c[2 * j + 1], mode) for j in range(len(c) // 2)])
    return lv
