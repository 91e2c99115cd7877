"""Python cross-oracle for the batched sum-check prover (tiny k only).

TEST INFRASTRUCTURE ONLY -- never imported by the product path.

A third, independent implementation of SURVEY.md Sec. 8(c.2) with Python
exact integers and ``hashlib``; it shares no code with ``oracle/oracle.c`` nor
with the CUDA path.  It also holds the *definition-level* checks that pin the
oracle (Sec. 2.3 for H; Alg. 1 for the round
structure):

* ``hypercube_sum``      -- H = sum_{x in {0,1}^k} prod_m f_m(x)
* ``mle``                -- f(z) = sum_y T[y] * eq(y, z), the plain multilinear
                            extension with index b = sum b_i 2^{i-1}
* ``round_poly_direct``  -- g_i(X) straight from its definition (sum over the
                            unbound Boolean variables of prod_m f_m evaluated
                            at the bound challenges), no folding at all.
* ``prove``              -- the fold algorithm, step by step.
* ``alg1``               -- Algorithm 1 of the paper, literally.
* ``verify``             -- the O(n) verifier.
"""
from __future__ import annotations

import hashlib
import itertools

# BN254 scalar field modulus (reading R1 in DESIGN.md)
P = 0x30644E72E131A029B85045B68181585D2833E84879B9709143E1F593F0000001

ORDER_LSB = 0
ORDER_MSB = 1


def le256(x: int) -> bytes:
    return int(x).to_bytes(32, "little")


def transcript_init(seed: bytes, index: int, k: int, d: int, order: int) -> bytes:
    """state_0 = SHA-256(tag || seed || LE64 I || LE16 k || LE16 d || LE16 order || LE16 0)."""
    assert len(seed) == 32
    msg = (b"BZK-SUMCHECK-V1\x00" + seed + index.to_bytes(8, "little") + k.to_bytes(2, "little")
           + d.to_bytes(2, "little") + order.to_bytes(2, "little") + b"\x00\x00")
    assert len(msg) == 64
    return hashlib.sha256(msg).digest()


def transcript_round(state: bytes, g: list[int]) -> tuple[bytes, int]:
    """state_i = SHA-256(state_{i-1} || LE256 g(0) || ... || LE256 g(d)); r_i = LE(state_i) mod p."""
    st = hashlib.sha256(state + b"".join(le256(v) for v in g)).digest()
    return st, int.from_bytes(st, "little") % P


def pair(T: list[int], j: int, h: int, order: int) -> tuple[int, int]:
    return (T[2 * j], T[2 * j + 1]) if order == ORDER_LSB else (T[j], T[j + h])


def prove(tables: list[list[int]], k: int, seed: bytes, index: int, order: int = ORDER_LSB):
    """Fold algorithm. tables: d lists of 2^k ints < p.

    Returns (round_evals [k][d+1], challenges [k], finals [d], H)."""
    d = len(tables)
    T = [list(t) for t in tables]
    n = 1 << k
    assert all(len(t) == n for t in T)
    H = 0
    for x in range(n):
        prod = 1
        for m in range(d):
            prod = prod * T[m][x] % P
        H = (H + prod) % P
    state = transcript_init(seed, index, k, d, order)
    evals, chals = [], []
    size = n
    for _i in range(1, k + 1):
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
        state, r = transcript_round(state, g)
        evals.append(g)
        chals.append(r)
        for m in range(d):
            new = []
            for j in range(h):
                a, b = pair(T[m], j, h, order)
                new.append((a + r * (b - a)) % P)
            T[m] = new
        size = h
    finals = [T[m][0] for m in range(d)]
    return evals, chals, finals, H


def alg1(A: list[int], r: list[int]) -> list[tuple[int, int]]:
    """PAPER.md:111 Algorithm 1, line by line (d = 1, challenges given)."""
    A = list(A)
    n = len(r)
    assert len(A) == 1 << n
    pi = []
    for i in range(1, n + 1):                       # line 1
        p1 = p2 = 0
        h = 1 << (n - i)
        for b in range(h):                          # line 2
            p1 = (p1 + A[b]) % P                    # line 3
            p2 = (p2 + A[b + h]) % P                # line 4
            A[b] = ((1 - r[i - 1]) * A[b] + r[i - 1] * A[b + h]) % P   # line 5
        pi.append((p1, p2))
    return pi


def lagrange_eval(g: list[int], x: int) -> int:
    """g(x) from values at nodes 0..d."""
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


def verify(k, d, order, seed, index, evals, chals, finals, H) -> tuple[bool, str]:
    claim = H % P
    state = transcript_init(seed, index, k, d, order)
    for i in range(k):
        g = evals[i]
        if len(g) != d + 1 or any(not (0 <= v < P) for v in g):
            return False, f"round {i + 1}: malformed"
        if (g[0] + g[1]) % P != claim:
            return False, f"round {i + 1}: g(0)+g(1) != claim"
        state, r = transcript_round(state, g)
        if r != chals[i]:
            return False, f"round {i + 1}: challenge mismatch"
        claim = lagrange_eval(g, r)
    prod = 1
    for f in finals:
        prod = prod * f % P
    if prod != claim:
        return False, "final: prod f_m(rho) != claim"
    return True, "ok"


# ---------------------------------------------------------------- definitions

def eq_poly(y: int, z: list[int]) -> int:
    """eq(y, z) = prod_l (y_l z_l + (1 - y_l)(1 - z_l)), y_l = bit l-1 of y."""
    acc = 1
    for l, zl in enumerate(z):
        yl = (y >> l) & 1
        acc = acc * (zl if yl else (1 - zl)) % P
    return acc


def mle(T: list[int], z: list[int]) -> int:
    """Multilinear extension at z = (z_1..z_k): sum_y T[y] eq(y, z)."""
    assert len(T) == 1 << len(z)
    return sum(T[y] * eq_poly(y, z) for y in range(len(T))) % P


def hypercube_sum(tables: list[list[int]]) -> int:
    n = len(tables[0])
    acc = 0
    for x in range(n):
        prod = 1
        for t in tables:
            prod = prod * t[x] % P
        acc = (acc + prod) % P
    return acc


def bound_var(i: int, k: int, order: int) -> int:
    """0-based index of the variable bound in round i (1-based): LSB x_i, MSB x_{k-i+1}."""
    return i - 1 if order == ORDER_LSB else k - i


def round_poly_direct(tables, k, chals_before: list[int], X: int, order: int) -> int:
    """g_i(X) by definition, i = len(chals_before)+1: sum over the unbound Boolean
    variables of prod_m f_m(point), point built from challenges, X and the Booleans."""
    i = len(chals_before) + 1
    fixed = {bound_var(j + 1, k, order): chals_before[j] for j in range(i - 1)}
    fixed[bound_var(i, k, order)] = X
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


def rho_point(chals: list[int], k: int, order: int) -> list[int]:
    """rho assigns r_i to x_{sigma(i)}; returned as (z_1..z_k)."""
    z = [0] * k
    for i, r in enumerate(chals, start=1):
        z[bound_var(i, k, order)] = r
    return z
