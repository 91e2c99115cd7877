"""Pins for the linear-time encoder oracle (readings R21-R24), -m "not gpu".

The C oracle (orc_encode) is checked against things other than itself:
* a Python cross-oracle on dense integer matrices built from the CSR inputs (bit-exact);
* linearity over F_p: Enc(a x + b y) = a Enc(x) + b Enc(y) (the code is linear);
* the structure of P:113-117 by independent dense products: codeword = x || z || B z with
  z = Enc(A x) at the next level, and x || G0 x at the base;
* injectivity: the generator matrix (encodings of the unit vectors) has full rank n over F_p;
* the graph inputs: left-regular (every left vertex has exactly c / d distinct right neighbours),
  nonzero canonical weights, rows = right vertices;
* a golden digest written by tests/golden/make_golden_encoder.py from oracle/ only.
"""
import hashlib
import os
import random

import numpy as np
import pytest

import oracle
from oracle.py import encoder as pye
from paper_conf_asplos_lucw0cz25_b200 import inputs

P = pye.P
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def ints(a):
    return oracle.from_limbs(a)


def msg(n, seed):
    return inputs.gen_tables(1, 1, n.bit_length() - 1, first_index=seed)[0, 0]


@pytest.mark.parametrize("log_n", [6, 7, 8, 10])
def test_c_oracle_equals_python_dense_cross_oracle(log_n):
    code = inputs.gen_code(log_n, 6)
    x = msg(1 << log_n, log_n)
    got = ints(oracle.encode(code, x))
    assert got == pye.encode(code, ints(x))


def test_linearity():
    code = inputs.gen_code(9, 6)
    n = 1 << 9
    x, y = ints(msg(n, 1)), ints(msg(n, 2))
    a, b = 0x1234567 % P, (P - 987654321) % P
    comb = [(a * u + b * v) % P for u, v in zip(x, y)]
    ex = ints(oracle.encode(code, oracle.to_limbs(x)))
    ey = ints(oracle.encode(code, oracle.to_limbs(y)))
    ec = ints(oracle.encode(code, oracle.to_limbs(comb)))
    assert ec == [(a * u + b * v) % P for u, v in zip(ex, ey)]


def test_structure_by_dense_products():
    code = inputs.gen_code(10, 6)
    n = 1 << 10
    x = ints(msg(n, 3))
    c = ints(oracle.encode(code, oracle.to_limbs(x)))
    assert len(c) == 2 * n and c[:n] == x
    A0, B0 = pye.dense(code["A"][0]), pye.dense(code["B"][0])
    y = pye.matvec(A0, x)
    z = c[n:n + n // 2]
    # z is the next level's codeword of y: systematic prefix y, then its own (z', w') parts
    assert z[:n // 4] == y
    assert c[n + n // 2:] == pye.matvec(B0, z)
    # and the next level's own structure
    A1, B1 = pye.dense(code["A"][1]), pye.dense(code["B"][1])
    y1 = pye.matvec(A1, y)
    z1 = z[n // 4:n // 4 + n // 8]
    assert z1[:n // 16] == y1 and z[n // 4 + n // 8:] == pye.matvec(B1, z1)
    # base level: x_L || G0 x_L
    G = pye.dense(code["G0"])
    assert z1[n // 16:] == pye.matvec(G, y1)


@pytest.mark.parametrize("log_n", [6, 7])
def test_generator_matrix_full_rank(log_n):
    code = inputs.gen_code(log_n, 6)
    n = 1 << log_n
    rows = []
    for i in range(n):
        e = [0] * n
        e[i] = 1
        rows.append(ints(oracle.encode(code, oracle.to_limbs(e))))
    assert pye.rank_mod_p(rows) == n


def test_graph_inputs_are_left_regular_and_canonical():
    code = inputs.gen_code(12, 6)
    assert code["levels"] == 3 and code["m"] == 64
    for l in range(code["levels"]):
        for M, deg, rows, cols in ((code["A"][l], inputs.ENC_C, (1 << (12 - 2 * l)) // 4, 1 << (12 - 2 * l)),
                                   (code["B"][l], inputs.ENC_D, (1 << (12 - 2 * l)) // 2, (1 << (12 - 2 * l)) // 2)):
            assert M["rows"] == rows and M["cols"] == cols and M["row_ptr"][-1] == deg * cols
            r = np.repeat(np.arange(rows), np.diff(M["row_ptr"].astype(np.int64)))
            pairs = set(zip(r.tolist(), M["col"].tolist()))
            assert len(pairs) == deg * cols                       # distinct right neighbours
            assert np.all(np.bincount(M["col"], minlength=cols) == deg)   # left-regular
            v = ints(M["val"])
            assert all(0 < w < P for w in v)


def test_non_canonical_message_rejected():
    code = inputs.gen_code(6, 6)
    x = msg(64, 0).copy()
    x[5] = oracle.to_limbs([P])[0]
    with pytest.raises(ValueError):
        oracle.encode(code, x)


def test_batch_equals_single():
    code = inputs.gen_code(8, 6)
    ms = inputs.gen_tables(3, 1, 8, first_index=4)[:, 0]
    out = oracle.encode_batch(code, ms, nthreads=2)
    for b in range(3):
        assert np.array_equal(out[b], oracle.encode(code, ms[b]))


def test_golden_encoder_digest():
    rows = []
    with open(os.path.join(GOLDEN, "encoder_small.txt")) as f:
        rows = [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]
    assert len(rows) >= 3
    for log_n, idx, digest in rows:
        code = inputs.gen_code(int(log_n), 6)
        c = oracle.encode(code, msg(1 << int(log_n), int(idx)))
        assert hashlib.sha256(c.astype("<u8").tobytes()).hexdigest() == digest
