"""CPU oracle for the batched sum-check prover -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_asplos_lucw0cz25_b200``) never imports it and shares no code with it.

``liboracle.so`` is compiled from ``oracle/oracle.c`` by :func:`build` (plain
``gcc -O2``; building the checker is not using it).  See oracle.c's header for
what each function follows in PAPER.md.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

P = 0x30644E72E131A029B85045B68181585D2833E84879B9709143E1F593F0000001


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               "-o", _LIB, _SRC])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u8p = ctypes.c_char_p
        u64p = ctypes.POINTER(ctypes.c_uint64)
        u32, u64 = ctypes.c_uint32, ctypes.c_uint64
        L.orc_prove.argtypes = [u32, u32, u32, u8p, u64, u64p, u64p, u64p, u64p, u64p]
        L.orc_prove_batch.argtypes = [u32, u32, u32, u8p, u64, u64, u64p, u64p, u64p, u64p, u64p,
                                      ctypes.c_int]
        L.orc_alg1.argtypes = [u32, u64p, u64p, u64p]
        L.orc_prove_given.argtypes = [u32, u32, u32, u64p, u64p, u64p, u64p, u64p, u64p]
        L.orc_verify.argtypes = [u32, u32, u32, u8p, u64, u64p, u64p, u64p, u64p]
        L.orc_mle.argtypes = [u32, u64p, u64p, u64p]
        L.orc_hsum.argtypes = [u32, u32, u64p, u64p]
        L.orc_fr_op.argtypes = [ctypes.c_int, u64, u64p, u64p, u64p]
        L.orc_sha256.argtypes = [u8p, u64, ctypes.c_char_p]
        L.orc_mu.argtypes = [u64p]
        L.orc_gl_prove.argtypes = [u32, u32, u32, u8p, u64, u64p, u64p, u64p, u64p, u64p, u64p]
        L.orc_gl_op.argtypes = [ctypes.c_int, u64, u64p, u64p, u64p]
        vp = ctypes.c_void_p
        L.orc_sha256_compress.argtypes = [vp, vp, vp]
        L.orc_merkle.argtypes = [u32, ctypes.c_int, vp, vp, vp]
        L.orc_merkle_batch.argtypes = [u32, ctypes.c_int, u64, vp, vp, vp, ctypes.c_int]
        L.orc_merkle_path.argtypes = [u32, vp, u64, vp]
        L.orc_merkle_verify_path.argtypes = [u32, ctypes.c_int, vp, u64, vp, vp]
        L.orc_encode.argtypes = [u32, u32, vp, vp, vp, vp, vp]
        L.orc_encode_batch.argtypes = [u32, u32, vp, vp, vp, u64, vp, vp, ctypes.c_int]
        _lib = L
    return _lib


def _p(a: np.ndarray | None):
    if a is None:
        return None
    assert a.dtype == np.uint64 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


# ---------------------------------------------------------------- conversions

def to_limbs(values) -> np.ndarray:
    """Python ints -> [n][4] uint64 little-endian limbs."""
    vals = list(values)
    out = np.zeros((len(vals), 4), dtype=np.uint64)
    for i, v in enumerate(vals):
        for w in range(4):
            out[i, w] = (v >> (64 * w)) & 0xFFFFFFFFFFFFFFFF
    return out


def from_limbs(a: np.ndarray) -> list[int]:
    a = np.ascontiguousarray(a, dtype=np.uint64).reshape(-1, 4)
    return [int(r[0]) | (int(r[1]) << 64) | (int(r[2]) << 128) | (int(r[3]) << 192) for r in a]


# ---------------------------------------------------------------- API

def prove(tables: np.ndarray, k: int, d: int, order: int, seed: bytes, index: int):
    """One proof.  tables: uint64 [d][2^k][4].  Returns dict of uint64 arrays."""
    tables = np.ascontiguousarray(tables, dtype=np.uint64)
    assert tables.shape == (d, 1 << k, 4)
    ev = np.zeros((k, d + 1, 4), np.uint64)
    ch = np.zeros((k, 4), np.uint64)
    fi = np.zeros((d, 4), np.uint64)
    cl = np.zeros((4,), np.uint64)
    s = lib().orc_prove(k, d, order, seed, index, _p(tables), _p(ev), _p(ch), _p(fi), _p(cl))
    if s:
        raise ValueError(f"orc_prove failed: {s}")
    return {"round_evals": ev, "challenges": ch, "final_evals": fi, "claims": cl}


def prove_given(tables: np.ndarray, k: int, d: int, order: int, challenges: np.ndarray):
    """Paper-literal mode (Alg. 1): challenges [k][4] are inputs."""
    tables = np.ascontiguousarray(tables, dtype=np.uint64)
    challenges = np.ascontiguousarray(challenges, dtype=np.uint64)
    assert tables.shape == (d, 1 << k, 4) and challenges.shape == (k, 4)
    ev = np.zeros((k, d + 1, 4), np.uint64)
    ch = np.zeros((k, 4), np.uint64)
    fi = np.zeros((d, 4), np.uint64)
    cl = np.zeros((4,), np.uint64)
    s = lib().orc_prove_given(k, d, order, _p(tables), _p(challenges), _p(ev), _p(ch), _p(fi), _p(cl))
    if s:
        raise ValueError(f"orc_prove_given failed: {s}")
    return {"round_evals": ev, "challenges": ch, "final_evals": fi, "claims": cl}


def prove_batch(tables: np.ndarray, k: int, d: int, order: int, seed: bytes, first_index: int,
                nthreads: int | None = None):
    """Batch: tables uint64 [B][d][2^k][4] -> dict of [B]-leading arrays."""
    tables = np.ascontiguousarray(tables, dtype=np.uint64)
    B = tables.shape[0]
    assert tables.shape == (B, d, 1 << k, 4)
    ev = np.zeros((B, k, d + 1, 4), np.uint64)
    ch = np.zeros((B, k, 4), np.uint64)
    fi = np.zeros((B, d, 4), np.uint64)
    cl = np.zeros((B, 4), np.uint64)
    if nthreads is None:
        nthreads = min(B, len(os.sched_getaffinity(0))) or 1
    s = lib().orc_prove_batch(k, d, order, seed, first_index, B, _p(tables), _p(ev), _p(ch),
                              _p(fi), _p(cl), nthreads)
    if s:
        raise ValueError(f"orc_prove_batch failed: {s}")
    return {"round_evals": ev, "challenges": ch, "final_evals": fi, "claims": cl}


def verify(k, d, order, seed, index, round_evals, challenges, final_evals, claim) -> int:
    a = [np.ascontiguousarray(x, dtype=np.uint64) for x in (round_evals, challenges, final_evals, claim)]
    return lib().orc_verify(k, d, order, seed, index, *[_p(x) for x in a])


def alg1(A: np.ndarray, r: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.uint64)
    r = np.ascontiguousarray(r, dtype=np.uint64)
    n = r.shape[0]
    out = np.zeros((n, 2, 4), np.uint64)
    s = lib().orc_alg1(n, _p(A), _p(r), _p(out))
    if s:
        raise ValueError(f"orc_alg1 failed: {s}")
    return out


def mle(table: np.ndarray, point: np.ndarray) -> np.ndarray:
    table = np.ascontiguousarray(table, dtype=np.uint64)
    point = np.ascontiguousarray(point, dtype=np.uint64)
    k = point.shape[0]
    out = np.zeros(4, np.uint64)
    lib().orc_mle(k, _p(table), _p(point), _p(out))
    return out


def hsum(tables: np.ndarray, k: int, d: int) -> np.ndarray:
    tables = np.ascontiguousarray(tables, dtype=np.uint64)
    out = np.zeros(4, np.uint64)
    lib().orc_hsum(k, d, _p(tables), _p(out))
    return out


def fr_op(op: str, a: np.ndarray, b: np.ndarray | None = None) -> np.ndarray:
    code = {"add": 0, "sub": 1, "mul": 2, "inv": 3, "reduce": 4}[op]
    a = np.ascontiguousarray(a, dtype=np.uint64)
    b = None if b is None else np.ascontiguousarray(b, dtype=np.uint64)
    out = np.zeros_like(a)
    lib().orc_fr_op(code, a.shape[0], _p(a), _p(b), _p(out))
    return out


def sha256(msg: bytes) -> bytes:
    out = ctypes.create_string_buffer(32)
    lib().orc_sha256(msg, len(msg), out)
    return out.raw


def mu() -> int:
    out = np.zeros(5, np.uint64)
    lib().orc_mu(_p(out))
    return sum(int(out[i]) << (64 * i) for i in range(5))


# ---------------------------------------------------------------- Goldilocks (NEXT-2, reading R15)

PGL = 0xFFFFFFFF00000001


def gl_prove(tables: np.ndarray, k: int, d: int, order: int, seed: bytes, index: int, given=None):
    """One Goldilocks proof.  tables: uint64 [d][2^k].  given: optional challenges [k] (Alg. 1 mode)."""
    tables = np.ascontiguousarray(tables, dtype=np.uint64)
    assert tables.shape == (d, 1 << k)
    ev = np.zeros((k, d + 1), np.uint64)
    ch = np.zeros((k,), np.uint64)
    fi = np.zeros((d,), np.uint64)
    cl = np.zeros((1,), np.uint64)
    g = None if given is None else np.ascontiguousarray(given, dtype=np.uint64)
    s = lib().orc_gl_prove(k, d, order, seed, index, _p(tables), _p(g), _p(ev), _p(ch), _p(fi), _p(cl))
    if s:
        raise ValueError(f"orc_gl_prove failed: {s}")
    return {"round_evals": ev, "challenges": ch, "final_evals": fi, "claims": cl}


def gl_op(op: str, a: np.ndarray, b: np.ndarray) -> np.ndarray:
    code = {"add": 0, "sub": 1, "mul": 2}[op]
    a = np.ascontiguousarray(a, dtype=np.uint64)
    b = np.ascontiguousarray(b, dtype=np.uint64)
    out = np.zeros_like(a)
    lib().orc_gl_op(code, a.shape[0], _p(a), _p(b), _p(out))
    return out


# ---------------------------------------------------------------- Merkle trees (NEXT-3, readings R17-R19)

MERKLE_COMPRESS = 0   # H = one SHA-256 compression of the 512-bit block from the FIPS IV
MERKLE_FIPS = 1       # H = FIPS 180-4 SHA-256 of the 64-byte message


def _u8(a: np.ndarray):
    assert a.dtype == np.uint8 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def sha256_compress(state, block: bytes):
    """One SHA-256 compression: state = 8 uint32 words, block = 64 bytes -> 8 words."""
    h = np.ascontiguousarray(np.asarray(state, dtype=np.uint32))
    b = np.frombuffer(bytes(block), dtype=np.uint8).copy()
    assert h.shape == (8,) and b.shape == (64,)
    out = np.zeros(8, np.uint32)
    lib().orc_sha256_compress(h.ctypes.data, b.ctypes.data, out.ctypes.data)
    return [int(x) for x in out]


def merkle(blocks: np.ndarray, n: int, mode: int = MERKLE_COMPRESS, nodes: bool = True):
    """One tree: blocks uint8 [2^n][64] -> (root bytes, nodes uint8 [2^(n+1)-1][32] or None)."""
    blocks = np.ascontiguousarray(blocks, dtype=np.uint8).reshape(-1)
    assert blocks.size == (64 << n)
    root = np.zeros(32, np.uint8)
    nd = np.zeros(((2 << n) - 1) * 32, np.uint8) if nodes else None
    s = lib().orc_merkle(n, mode, _u8(blocks), None if nd is None else _u8(nd), _u8(root))
    if s:
        raise ValueError(f"orc_merkle failed: {s}")
    return root.tobytes(), (None if nd is None else nd.reshape(-1, 32))


def merkle_batch(blocks: np.ndarray, n: int, mode: int = MERKLE_COMPRESS, nodes: bool = False,
                 nthreads: int | None = None):
    """Batch: blocks uint8 [B][2^n][64] -> (roots uint8 [B][32], nodes uint8 [B][2^(n+1)-1][32] or None)."""
    blocks = np.ascontiguousarray(blocks, dtype=np.uint8)
    B = blocks.shape[0]
    assert blocks.size == B * (64 << n)
    roots = np.zeros((B, 32), np.uint8)
    nd = np.zeros((B, (2 << n) - 1, 32), np.uint8) if nodes else None
    if nthreads is None:
        nthreads = min(B, len(os.sched_getaffinity(0))) or 1
    s = lib().orc_merkle_batch(n, mode, B, _u8(blocks.reshape(-1)), None if nd is None else _u8(nd),
                               _u8(roots), nthreads)
    if s:
        raise ValueError(f"orc_merkle_batch failed: {s}")
    return roots, nd


def merkle_path(nodes: np.ndarray, n: int, x: int) -> np.ndarray:
    nodes = np.ascontiguousarray(nodes, dtype=np.uint8)
    path = np.zeros((max(n, 1), 32), np.uint8)
    lib().orc_merkle_path(n, _u8(nodes), x, _u8(path))
    return path[:n]


def merkle_verify_path(n: int, mode: int, block: bytes, x: int, path: np.ndarray, root: bytes) -> bool:
    b = np.frombuffer(bytes(block), dtype=np.uint8).copy()
    p = np.ascontiguousarray(path, dtype=np.uint8).reshape(-1)
    if p.size == 0:
        p = np.zeros(32, np.uint8)
    r = np.frombuffer(bytes(root), dtype=np.uint8).copy()
    return bool(lib().orc_merkle_verify_path(n, mode, _u8(b), x, _u8(p), _u8(r)))


# ---------------------------------------------------------------- linear-time encoder (NEXT-4, readings R21-R24)

class _Csr(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_uint32), ("cols", ctypes.c_uint32), ("row_ptr", ctypes.c_void_p),
                ("col", ctypes.c_void_p), ("val", ctypes.c_void_p)]


def _csr(m: dict) -> _Csr:
    for k_ in ("row_ptr", "col", "val"):
        assert m[k_].flags["C_CONTIGUOUS"]
    return _Csr(m["rows"], m["cols"], m["row_ptr"].ctypes.data, m["col"].ctypes.data, m["val"].ctypes.data)


def _code_args(code: dict):
    L = code["levels"]
    A = (_Csr * max(1, L))(*[_csr(a) for a in code["A"]])
    B = (_Csr * max(1, L))(*[_csr(b) for b in code["B"]])
    G0 = _csr(code["G0"])
    return A, B, G0


def encode(code: dict, msg: np.ndarray) -> np.ndarray:
    """One message [n][4] (canonical) -> codeword [2n][4] (oracle/oracle.c orc_encode)."""
    msg = np.ascontiguousarray(msg, dtype=np.uint64)
    n = 1 << code["log_n"]
    assert msg.shape == (n, 4)
    out = np.zeros((2 * n, 4), np.uint64)
    A, B, G0 = _code_args(code)
    s = lib().orc_encode(code["log_n"], code["levels"], ctypes.addressof(A), ctypes.addressof(B),
                         ctypes.addressof(G0), msg.ctypes.data, out.ctypes.data)
    if s:
        raise ValueError(f"orc_encode failed: {s}")
    return out


def encode_batch(code: dict, msgs: np.ndarray, nthreads: int | None = None) -> np.ndarray:
    msgs = np.ascontiguousarray(msgs, dtype=np.uint64)
    Bn = msgs.shape[0]
    n = 1 << code["log_n"]
    assert msgs.shape == (Bn, n, 4)
    out = np.zeros((Bn, 2 * n, 4), np.uint64)
    if nthreads is None:
        nthreads = min(Bn, len(os.sched_getaffinity(0))) or 1
    A, B, G0 = _code_args(code)
    s = lib().orc_encode_batch(code["log_n"], code["levels"], ctypes.addressof(A), ctypes.addressof(B),
                               ctypes.addressof(G0), Bn, msgs.ctypes.data, out.ctypes.data, nthreads)
    if s:
        raise ValueError(f"orc_encode_batch failed: {s}")
    return out


# ---------------------------------------------------------------- the section-4 chain (NEXT-4)

def commit_prove(code: dict, segments: np.ndarray, tables: np.ndarray, k: int, d: int, order: int, index: int,
                 mode: int = MERKLE_COMPRESS):
    """One proof of the chain of PAPER.md:207-213 (Sec. 4, Fig. 7), step by step:
    1. every message segment is encoded ("each encoded into an error-correction code");
    2. every codeword is committed with a Merkle tree over its bytes as 64-byte blocks;
    3. "these roots serve as leaf nodes for another Merkle tree module, ultimately yielding a single
       final root": level 1 = H(root_2j || root_2j+1), ..., one root (S = 1: the root itself);
    4. the sum-check's transcript is seeded with the final root (reading R25).
    segments: uint64 [S][n][4].  Returns (codewords [S][2n][4], roots [S][32], final root, proof dict)."""
    S = segments.shape[0]
    assert S >= 1 and S & (S - 1) == 0
    codes = np.stack([encode(code, segments[s]) for s in range(S)])
    roots = np.stack([np.frombuffer(merkle(codes[s].astype("<u8").view(np.uint8).reshape(-1, 64),
                                           code["log_n"], mode, nodes=False)[0], np.uint8) for s in range(S)])
    if S == 1:
        final = roots[0].tobytes()
    else:
        final = merkle(roots.reshape(S // 2, 64), (S // 2).bit_length() - 1, mode, nodes=False)[0]
    return codes, roots, final, prove(tables, k, d, order, final, index)
