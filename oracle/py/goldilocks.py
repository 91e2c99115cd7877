"""Python cross-oracle for the Goldilocks field instance (R15).

TEST INFRASTRUCTURE ONLY.  Python integers + hashlib; independent of oracle/oracle.c and of the
CUDA path.  Same prover as oracle/py/sumcheck.py (Alg. 1 generalised), over
p = 2^64 - 2^32 + 1 with the transcript framed by field id 1 and LE64-encoded evaluations.
"""
from __future__ import annotations

import hashlib
import itertools

P = 0xFFFFFFFF00000001


def transcript_init(seed: bytes, index: int, k: int, d: int, order: int) -> bytes:
    msg = (b"BZK-SUMCHECK-V1\x00" + seed + index.to_bytes(8, "little") + k.to_bytes(2, "little")
           + d.to_bytes(2, "little") + order.to_bytes(2, "little") + (1).to_bytes(2, "little"))
    assert len(msg) == 64
    return hashlib.sha256(msg).digest()


def transcript_round(state: bytes, g: list[int]) -> tuple[bytes, int]:
    st = hashlib.sha256(state + b"".join(int(v).to_bytes(8, "little") for v in g)).digest()
    return st, int.from_bytes(st[:8], "little") % P


def pair(T, j, h, order):
    return (T[2 * j], T[2 * j + 1]) if order == 0 else (T[j], T[j + h])


def prove(tables, k, seed, index, order=0, given=None):
    d = len(tables)
    T = [list(t) for t in tables]
    H = 0
    for x in range(1 << k):
        prod = 1
        for m in range(d):
            prod = prod * T[m][x] % P
        H = (H + prod) % P
    state = transcript_init(seed, index, k, d, order)
    evals, chals = [], []
    size = 1 << k
    for i in range(k):
        h = size // 2
        g = []
        for t in range(d + 1):
            acc = 0
            for j in range(h):
                prod = 1
                for m in range(d):
                    a, b = pair(T[m], j, h, order)
                    prod = prod * ((a + t * (b - a)) % P) % P
                acc = (acc + prod) % P
            g.append(acc)
        if given is None:
            state, r = transcript_round(state, g)
        else:
            r = given[i]
        evals.append(g)
        chals.append(r)
        for m in range(d):
            T[m] = [(a + r * (b - a)) % P for a, b in (pair(T[m], j, h, order) for j in range(h))]
        size = h
    return evals, chals, [T[m][0] for m in range(d)], H


def lagrange_eval(g, x):
    d = len(g) - 1
    acc = 0
    for j in range(d + 1):
        num, den = 1, 1
        for l in range(d + 1):
            if l != j:
                num = num * (x - l) % P
                den = den * (j - l) % P
        acc = (acc + g[j] * num * pow(den, P - 2, P)) % P
    return acc


def mle(T, z):
    acc = 0
    for y in range(len(T)):
        e = 1
        for l, zl in enumerate(z):
            e = e * (zl if (y >> l) & 1 else (1 - zl)) % P
        acc = (acc + T[y] * e) % P
    return acc


def round_poly_direct(tables, k, chals_before, X, order):
    i = len(chals_before) + 1
    bv = (lambda ii: ii - 1) if order == 0 else (lambda ii: k - ii)
    fixed = {bv(j + 1): chals_before[j] for j in range(i - 1)}
    fixed[bv(i)] = X
    free = [v for v in range(k) if v not in fixed]
    acc = 0
    for bits in itertools.product((0, 1), repeat=len(free)):
        z = [0] * k
        for v, val in fixed.items():
            z[v] = val % P
        for v, bit in zip(free, bits):
            z[v] = bit
        prod = 1
        for t in tables:
            prod = prod * mle(t, z) % P
        acc = (acc + prod) % P
    return acc
