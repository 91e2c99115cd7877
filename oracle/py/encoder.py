"""Python cross-oracle for the linear-time (Spielman-style) encoder -- tiny n only.

TEST INFRASTRUCTURE ONLY -- never imported by the product path.

Independent of oracle/oracle.c and of the CUDA path: Python exact integers, the graphs as DENSE
matrices built from the CSR inputs, and the recursion of P:113-117 (Sec. 2.4, Fig. 3):
    Enc_l(x) = x || G0 x                       at the base level l = L
    Enc_l(x) = x || z || B_l z,  z = Enc_{l+1}(A_l x)   otherwise.
"""
from __future__ import annotations

P = 0x30644E72E131A029B85045B68181585D2833E84879B9709143E1F593F0000001


def limbs_to_int(row) -> int:
    return int(row[0]) | (int(row[1]) << 64) | (int(row[2]) << 128) | (int(row[3]) << 192)


def dense(m: dict) -> list[list[int]]:
    """CSR (rows = right vertices, cols = left vertices) -> dense rows x cols matrix of ints."""
    M = [[0] * m["cols"] for _ in range(m["rows"])]
    rp, col, val = m["row_ptr"], m["col"], m["val"]
    for r in range(m["rows"]):
        for e in range(int(rp[r]), int(rp[r + 1])):
            M[r][int(col[e])] = limbs_to_int(val[e])
    return M


def matvec(M: list[list[int]], x: list[int]) -> list[int]:
    return [sum(a * b for a, b in zip(row, x)) % P for row in M]


def encode(code: dict, x: list[int], l: int = 0) -> list[int]:
    if l == code["levels"]:
        return list(x) + matvec(dense(code["G0"]), x)
    z = encode(code, matvec(dense(code["A"][l]), x), l + 1)
    return list(x) + z + matvec(dense(code["B"][l]), z)


def rank_mod_p(rows: list[list[int]]) -> int:
    """Rank over F_p by Gaussian elimination."""
    M = [list(r) for r in rows]
    rank, ncols = 0, len(M[0]) if M else 0
    for c in range(ncols):
        piv = next((i for i in range(rank, len(M)) if M[i][c] % P), None)
        if piv is None:
            continue
        M[rank], M[piv] = M[piv], M[rank]
        inv = pow(M[rank][c], P - 2, P)
        M[rank] = [v * inv % P for v in M[rank]]
        for i in range(len(M)):
            if i != rank and M[i][c]:
                f = M[i][c]
                M[i] = [(a - f * b) % P for a, b in zip(M[i], M[rank])]
        rank += 1
    return rank
