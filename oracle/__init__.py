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
