"""Pins for the CPU oracle (-m "not gpu").

Each test checks the oracle against something other than itself: Python exact
integers, FIPS 180-4 vectors / hashlib, the plain definition of the sum-check
statement (Sec. 2.3), Algorithm 1 literally, the
multilinear extension via eq-polynomials, closed forms and a verifier.
"""
import hashlib
import os
import random

import numpy as np
import pytest

from oracle.py import sumcheck as py
from paper_conf_asplos_lucw0cz25_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
P = py.P
SEED = inputs.DEFAULT_SEED


def read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def ints(a):
    from oracle import from_limbs
    return from_limbs(a)


# ---------------------------------------------------------------- field

def is_probable_prime(n):
    if n < 2:
        return False
    d, s = n - 1, 0
    while d % 2 == 0:
        d //= 2
        s += 1
    rng = random.Random(7)
    for _ in range(40):
        a = rng.randrange(2, n - 1)
        x = pow(a, d, n)
        if x in (1, n - 1):
            continue
        for _ in range(s - 1):
            x = x * x % n
            if x == n - 1:
                break
        else:
            return False
    return True


def test_modulus_is_bn254_r():
    g = dict((r[0], r[1]) for r in read_golden("bn254_fr.txt"))
    u = int(g["u"])
    r = 36 * u**4 + 36 * u**3 + 18 * u**2 + 6 * u + 1
    assert r == int(g["p"], 16) == P
    assert P.bit_length() == int(g["bits"])
    two = int(g["two_adicity"])
    assert (P - 1) % (1 << two) == 0 and (P - 1) % (1 << (two + 1)) != 0
    assert is_probable_prime(P)
    assert 4 * P < 2**256 and P > 2**253


def test_barrett_mu(orc):
    assert orc.mu() == 2**512 // P


def _edge_values():
    return [0, 1, 2, P - 1, P - 2, 2**253, 2**253 - 1, (2**256) % P, (2**64) % P, 2**192, P // 2,
            (P + 1) // 2, 0xFFFFFFFF, 0xFFFFFFFFFFFFFFFF, 2**128 - 1]


def test_field_ops_vs_python_ints(orc):
    rng = random.Random(1)
    n = 20000
    a = [rng.randrange(P) for _ in range(n)] + _edge_values() * len(_edge_values())
    e = _edge_values()
    b = [rng.randrange(P) for _ in range(n)] + [x for x in e for _ in e]
    A, B = orc.to_limbs(a), orc.to_limbs(b)
    assert ints(orc.fr_op("add", A, B)) == [(x + y) % P for x, y in zip(a, b)]
    assert ints(orc.fr_op("sub", A, B)) == [(x - y) % P for x, y in zip(a, b)]
    assert ints(orc.fr_op("mul", A, B)) == [(x * y) % P for x, y in zip(a, b)]
    nz = [x for x in a[:500] if x]
    assert ints(orc.fr_op("inv", orc.to_limbs(nz))) == [pow(x, P - 2, P) for x in nz]


def test_reduce_256_bit(orc):
    rng = random.Random(2)
    v = [rng.randrange(2**256) for _ in range(5000)] + [2**256 - 1, 5 * P, 5 * P - 1, ((2**256 - 1) // P) * P, P, 0]
    assert ints(orc.fr_op("reduce", orc.to_limbs(v))) == [x % P for x in v]


# ---------------------------------------------------------------- SHA-256

def test_sha256_fips_vectors(orc):
    for spec, digest in read_golden("sha256_fips180_4.txt"):
        if spec.startswith("rep:"):
            _, cnt, txt = spec.split(":", 2)
            msg = txt.encode() * int(cnt)
        else:
            msg = spec.encode()
        assert orc.sha256(msg).hex() == digest
        assert hashlib.sha256(msg).hexdigest() == digest


def test_sha256_vs_hashlib_all_padding_edges(orc):
    rng = random.Random(3)
    for n in list(range(0, 300)):
        msg = bytes(rng.randrange(256) for _ in range(n))
        assert orc.sha256(msg) == hashlib.sha256(msg).digest(), n


# ---------------------------------------------------------------- inputs generator

def test_splitmix64_reference_value():
    # SplitMix64 (Steele, Lea, Flood 2014) seeded with state 0: first output is 0xe220a8397b1dcdaf
    v = inputs.splitmix64(np.array([0], dtype=np.uint64), data_seed=0)
    assert int(v[0]) == 0xE220A8397B1DCDAF


def test_generator_properties():
    t = inputs.gen_tables(3, 2, 5, first_index=10)
    assert t.shape == (3, 2, 32, 4)
    vals = ints(t)
    assert all(v < P for v in vals)      # canonical over the whole field (SURVEY 8(d) recipe)
    assert len(set(vals)) == len(vals)
    # independent of batch composition: proof 11 generated alone is identical
    assert np.array_equal(inputs.gen_tables(1, 2, 5, first_index=11)[0], t[1])
    s = inputs.gen_tables(2, 3, 4, dist="smallint")
    assert all(v < 256 for v in ints(s))
    vml = inputs.gen_tables(1, 2, 4, dist="vml")
    assert all(v < 256 for v in ints(vml[0, 0])) and max(ints(vml[0, 1])) > 2**200


# ---------------------------------------------------------------- prover

def _tables_py(t):
    return [ints(t[m]) for m in range(t.shape[0])]


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3, 4])
@pytest.mark.parametrize("k", [0, 1, 2, 3, 5])
def test_c_oracle_equals_python_cross_oracle(orc, k, d, order):
    t = inputs.gen_tables(1, d, k, first_index=7 + k)[0]
    out = orc.prove(t, k, d, order, SEED, 7 + k)
    ev, ch, fi, H = py.prove(_tables_py(t), k, SEED, 7 + k, order)
    assert [ints(out["round_evals"][i]) for i in range(k)] == ev
    assert ints(out["challenges"]) == ch
    assert ints(out["final_evals"]) == fi
    assert ints(out["claims"])[0] == H


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3, 4])
def test_claim_is_hypercube_sum(orc, d, order):
    k = 6
    t = inputs.gen_tables(1, d, k, first_index=3)[0]
    out = orc.prove(t, k, d, order, SEED, 3)
    H = py.hypercube_sum(_tables_py(t))
    g1 = ints(out["round_evals"][0])
    assert (g1[0] + g1[1]) % P == H
    assert ints(out["claims"])[0] == H
    assert ints(orc.hsum(t, k, d))[0] == H


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3])
def test_round_invariant_and_final_check(orc, d, order):
    k = 8
    t = inputs.gen_tables(1, d, k, first_index=99)[0]
    out = orc.prove(t, k, d, order, SEED, 99)
    ev = [ints(out["round_evals"][i]) for i in range(k)]
    ch = ints(out["challenges"])
    fi = ints(out["final_evals"])
    claim = ints(out["claims"])[0]
    for i in range(k):
        assert (ev[i][0] + ev[i][1]) % P == claim, i
        claim = py.lagrange_eval(ev[i], ch[i])
    prod = 1
    for f in fi:
        prod = prod * f % P
    assert prod == claim


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3])
def test_round_poly_by_definition_incl_extra_node(orc, d, order):
    """g_i(t) for t = 0..d+1 straight from the definition (no folding); t = d+1 pins the nodes
    0..d and deg g_i <= d through Lagrange extrapolation."""
    k = 4
    t = inputs.gen_tables(1, d, k, first_index=5)[0]
    out = orc.prove(t, k, d, order, SEED, 5)
    tabs = _tables_py(t)
    ch = ints(out["challenges"])
    for i in range(k):
        g = ints(out["round_evals"][i])
        for X in range(d + 1):
            assert py.round_poly_direct(tabs, k, ch[:i], X, order) == g[X], (i, X)
        extra = py.round_poly_direct(tabs, k, ch[:i], d + 1, order)
        assert extra == py.lagrange_eval(g, d + 1)


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2])
def test_final_evals_are_mle_at_rho(orc, d, order):
    k = 7
    t = inputs.gen_tables(1, d, k, first_index=1)[0]
    out = orc.prove(t, k, d, order, SEED, 1)
    ch = ints(out["challenges"])
    rho = py.rho_point(ch, k, order)
    for m in range(d):
        f = ints(out["final_evals"][m])[0]
        assert f == py.mle(ints(t[m]), rho)
        assert ints(orc.mle(t[m], orc.to_limbs(rho)))[0] == f
    # LSB and MSB differ (the pin distinguishes the orders)
    rho_other = py.rho_point(ch, k, 1 - order)
    assert py.mle(ints(t[0]), rho_other) != ints(out["final_evals"][0])[0]


def test_closed_form_constant_tables(orc):
    k, d = 6, 3
    c = [12345, P - 7, 2**200 + 3]
    t = orc.to_limbs([c[m] for m in range(d) for _ in range(1 << k)]).reshape(d, 1 << k, 4)
    out = orc.prove(t, k, d, 0, SEED, 0)
    prodc = c[0] * c[1] * c[2] % P
    for i in range(1, k + 1):
        g = ints(out["round_evals"][i - 1])
        assert g == [(1 << (k - i)) * prodc % P] * (d + 1)
    assert ints(out["final_evals"]) == c


@pytest.mark.parametrize("order", [0, 1])
def test_closed_form_indicator_is_eq(orc, order):
    k = 6
    x0 = 0b101101
    T = [0] * (1 << k)
    T[x0] = 1
    out = orc.prove(orc.to_limbs(T).reshape(1, 1 << k, 4), k, 1, order, SEED, 4)
    rho = py.rho_point(ints(out["challenges"]), k, order)
    expect = 1
    for l in range(k):
        bit = (x0 >> l) & 1
        expect = expect * (rho[l] if bit else (1 - rho[l])) % P
    assert ints(out["final_evals"])[0] == expect


def test_closed_form_identity_table(orc):
    k = 10
    T = list(range(1 << k))
    out = orc.prove(orc.to_limbs(T).reshape(1, 1 << k, 4), k, 1, 0, SEED, 0)
    g1 = ints(out["round_evals"][0])
    assert (g1[0] + g1[1]) % P == (1 << (k - 1)) * ((1 << k) - 1)
    # LSB round 1 of T[x] = x: g_1(0) = sum of even x, g_1(1) = sum of odd x
    assert g1[0] == sum(range(0, 1 << k, 2)) and g1[1] == sum(range(1, 1 << k, 2))


def test_alg1_literal_equals_fold_prover(orc):
    """PAPER.md:111 Alg. 1 (d=1, pairs (b, b+2^{n-i}), two-mult update, given r's) reproduces
    (g_i(0), g_i(1)) of the MSB prover fed the same challenges."""
    n = 9
    t = inputs.gen_tables(1, 1, n, first_index=2)[0]
    out = orc.prove(t, n, 1, 1, SEED, 2)
    pi = orc.alg1(t[0], out["challenges"])
    assert np.array_equal(pi, out["round_evals"])
    A = ints(t[0])
    assert py.alg1(A, ints(out["challenges"])) == [tuple(ints(out["round_evals"][i])) for i in range(n)]


def test_k0_edge_case(orc):
    d = 3
    t = inputs.gen_tables(1, d, 0)[0]
    out = orc.prove(t, 0, d, 0, SEED, 0)
    v = ints(t.reshape(-1, 4))
    assert ints(out["final_evals"]) == v
    assert ints(out["claims"])[0] == v[0] * v[1] * v[2] % P
    assert orc.verify(0, d, 0, SEED, 0, out["round_evals"], out["challenges"], out["final_evals"],
                      out["claims"]) == 0


def test_non_canonical_input_rejected(orc):
    t = inputs.gen_tables(1, 1, 3)[0]
    t[0, 5] = orc.to_limbs([P])[0]
    with pytest.raises(ValueError):
        orc.prove(t, 3, 1, 0, SEED, 0)


def test_batch_equals_single_and_index_binds(orc):
    k, d = 5, 2
    tb = inputs.gen_tables(4, d, k, first_index=20)
    out = orc.prove_batch(tb, k, d, 0, SEED, 20, nthreads=3)
    for b in range(4):
        one = orc.prove(tb[b], k, d, 0, SEED, 20 + b)
        for key in one:
            assert np.array_equal(one[key], out[key][b])
    other = orc.prove(tb[0], k, d, 0, SEED, 21)
    assert not np.array_equal(other["challenges"], out["challenges"][0])
    seed2 = bytes([1]) + SEED[1:]
    other = orc.prove(tb[0], k, d, 0, seed2, 20)
    assert not np.array_equal(other["challenges"], out["challenges"][0])


@pytest.mark.parametrize("order", [0, 1])
def test_verifier_accepts_and_rejects_every_byte_mutation(orc, order):
    k, d = 3, 2
    t = inputs.gen_tables(1, d, k, first_index=8)[0]
    out = orc.prove(t, k, d, order, SEED, 8)
    args = [out["round_evals"], out["challenges"], out["final_evals"], out["claims"]]
    assert orc.verify(k, d, order, SEED, 8, *args) == 0
    ok, _ = py.verify(k, d, order, SEED, 8, [ints(out["round_evals"][i]) for i in range(k)],
                      ints(out["challenges"]), ints(out["final_evals"]), ints(out["claims"])[0])
    assert ok
    for ai in range(4):
        flat = args[ai].view(np.uint8).reshape(-1)
        for byte in range(flat.size):
            mut = [a.copy() for a in args]
            mut[ai].view(np.uint8).reshape(-1)[byte] ^= 0x01
            assert orc.verify(k, d, order, SEED, 8, *mut) != 0, (ai, byte)
    # wrong index / seed / order rejected
    assert orc.verify(k, d, order, SEED, 9, *args) != 0
    assert orc.verify(k, d, 1 - order, SEED, 8, *args) != 0


def test_golden_proof_regression(orc):
    """tests/golden/proof_small.txt was written by tests/golden/make_golden.py, which calls only
    oracle/ (never the CUDA path); it freezes the transcript bytes of reading R5-R7."""
    rows = read_golden("proof_small.txt")
    cur = {}
    for r in rows:
        if r[0] == "case":
            cur = dict(kv.split("=") for kv in r[1:])
            k, d, order, I = (int(cur[x]) for x in ("k", "d", "order", "index"))
            t = inputs.gen_tables(1, d, k, first_index=I, dist=cur.get("dist", "uniform"))[0]
            out = orc.prove(t, k, d, order, SEED, I)
        else:
            key, vals = r[0], [int(v, 16) for v in r[1:]]
            assert ints(out[key]) == vals, (cur, key)


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3])
def test_given_challenge_mode(orc, d, order):
    """Paper-literal mode (Alg. 1, r_i given): fed the Fiat-Shamir challenges it reproduces the FS
    proof; for d = 1, MSB it equals Alg. 1 line by line; with other challenges the round invariant
    and final check still hold."""
    k = 7
    t = inputs.gen_tables(1, d, k, first_index=12)[0]
    fs = orc.prove(t, k, d, order, SEED, 12)
    given = orc.prove_given(t, k, d, order, fs["challenges"])
    for key in fs:
        assert np.array_equal(given[key], fs[key]), key
    rng = np.random.default_rng(d)
    r = orc.to_limbs([int(x) * 0x9E3779B97F4A7C15 % P for x in rng.integers(1, 2**62, size=k)])
    out = orc.prove_given(t, k, d, order, r)
    assert np.array_equal(out["challenges"], r)
    if d == 1 and order == 1:
        assert np.array_equal(orc.alg1(t[0], r), out["round_evals"])
    ev = [ints(out["round_evals"][i]) for i in range(k)]
    claim = ints(out["claims"])[0]
    for i in range(k):
        assert (ev[i][0] + ev[i][1]) % P == claim
        claim = py.lagrange_eval(ev[i], ints(r)[i])
    prod = 1
    for f in ints(out["final_evals"]):
        prod = prod * f % P
    assert prod == claim
    rho = py.rho_point(ints(r), k, order)
    assert ints(out["final_evals"])[0] == py.mle(ints(t[0]), rho)


# ---------------------------------------------------------------- Goldilocks instance (NEXT-2)

from oracle.py import goldilocks as pgl  # noqa: E402

PGL = pgl.P


def test_goldilocks_modulus():
    assert PGL == 2**64 - 2**32 + 1
    assert is_probable_prime(PGL)
    assert (PGL - 1) % 2**32 == 0 and (PGL - 1) % 2**33 != 0     # 2-adicity 32
    assert pow(7, (PGL - 1) // 2, PGL) == PGL - 1                 # 7 is a non-residue (generator family)


def test_goldilocks_field_ops(orc):
    rng = np.random.default_rng(3)
    a = rng.integers(0, 2**63, size=5000, dtype=np.uint64) * np.uint64(2) + np.uint64(1)
    b = rng.integers(0, 2**63, size=5000, dtype=np.uint64)
    edge = np.array([0, 1, PGL - 1, 2**32, 2**32 - 1, 2**63, PGL - 2**32], dtype=np.uint64)
    a = np.concatenate([a, np.repeat(edge, len(edge))])
    b = np.concatenate([b, np.tile(edge, len(edge))])
    A, B = [int(x) % PGL for x in a], [int(x) % PGL for x in b]
    assert [int(x) for x in orc.gl_op("add", a, b)] == [(x + y) % PGL for x, y in zip(A, B)]
    assert [int(x) for x in orc.gl_op("sub", a, b)] == [(x - y) % PGL for x, y in zip(A, B)]
    assert [int(x) for x in orc.gl_op("mul", a, b)] == [(x * y) % PGL for x, y in zip(A, B)]


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d", [1, 2, 3])
def test_goldilocks_oracle_pins(orc, d, order):
    k = 5
    t = inputs.gen_tables_gl(1, d, k, first_index=3)[0]
    tabs = [[int(x) for x in t[m]] for m in range(d)]
    out = orc.gl_prove(t, k, d, order, SEED, 3)
    ev, ch, fi, H = pgl.prove(tabs, k, SEED, 3, order)
    assert [[int(x) for x in row] for row in out["round_evals"]] == ev            # C == Python
    assert [int(x) for x in out["challenges"]] == ch
    assert [int(x) for x in out["final_evals"]] == fi and int(out["claims"][0]) == H
    brute = 0
    for x in range(1 << k):
        prod = 1
        for m in range(d):
            prod = prod * tabs[m][x] % PGL
        brute = (brute + prod) % PGL
    assert H == brute and (ev[0][0] + ev[0][1]) % PGL == H
    claim = H
    for i in range(k):
        assert (ev[i][0] + ev[i][1]) % PGL == claim
        for X in (0, d + 1) if i < 3 else (0,):
            direct = pgl.round_poly_direct(tabs, k, ch[:i], X, order)
            assert direct == (ev[i][X] if X <= d else pgl.lagrange_eval(ev[i], X))
        claim = pgl.lagrange_eval(ev[i], ch[i])
    prod = 1
    for f in fi:
        prod = prod * f % PGL
    assert prod == claim
    z = [0] * k
    for i, r in enumerate(ch, start=1):
        z[i - 1 if order == 0 else k - i] = r
    assert fi[0] == pgl.mle(tabs[0], z)
    # paper-literal mode: fed the FS challenges it reproduces the proof
    giv = orc.gl_prove(t, k, d, order, SEED, 3, given=out["challenges"])
    for key in out:
        assert np.array_equal(giv[key], out[key])


def test_c5_golden_digests_file(orc):
    """tests/golden/c5_proof_digests.txt (written by make_golden_c5.py from oracle/ only) covers the
    8192 proofs of configs[1]/[4]; two of them recomputed here by the oracle."""
    import hashlib
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "c5_proof_digests.txt")
    rows = [ln.split() for ln in open(path) if ln.strip() and not ln.startswith("#")]
    assert [int(i) for i, _ in rows] == list(range(8192))
    gold = {int(i): d for i, d in rows}
    for i in (0, 8191):
        out = orc.prove(inputs.gen_tables(1, 2, 20, first_index=i)[0], 20, 2, 0, SEED, i)
        h = hashlib.sha256()
        for key in ("round_evals", "challenges", "final_evals", "claims"):
            h.update(out[key].astype("<u8").tobytes())
        assert h.hexdigest()[:16] == gold[i], i


@pytest.mark.parametrize("order", [0, 1])
def test_multiround_identity_reading_r26(order):
    """Reading R26, checked in plain Python integers against Algorithm 1 run round by
    round (oracle/py/sumcheck.py alg1 for MSB; the LSB fold for order 0): after m known-challenge rounds
    A'[y] = sum_z w(z) A[y, z] with w the eq-weights of r_1..r_m, and the rounds' sums are the
    w_{<i}-weighted column sums -- the identity k_multi evaluates."""
    from oracle.py import sumcheck as ps
    rnd = random.Random(26 + order)
    P = ps.P
    K, m = 7, 3
    A = [rnd.randrange(P) for _ in range(1 << K)]
    r = [rnd.randrange(P) for _ in range(m)]
    # reference: m rounds of Alg. 1 (MSB pairs b, b + h) or the LSB pairing (2j, 2j + 1)
    T, sums = list(A), []
    for i in range(m):
        h = len(T) // 2
        pairs = [(T[j], T[j + h]) if order == 1 else (T[2 * j], T[2 * j + 1]) for j in range(h)]
        sums.append((sum(a for a, _ in pairs) % P, sum(b for _, b in pairs) % P))
        T = [(a + r[i] * (b - a)) % P for a, b in pairs]
    if order == 1:
        assert [tuple(x) for x in ps.alg1(A, r + [0] * (K - m))[:m]] == sums
    # the identity
    Ny = 1 << (K - m)
    def bit(z, i):          # the bit of z bound in round i (1-based)
        return (z >> (m - i)) & 1 if order == 1 else (z >> (i - 1)) & 1
    def entry(y, z):
        return A[y + z * Ny] if order == 1 else A[(y << m) + z]
    def weight(z, upto):
        w = 1
        for i in range(1, upto + 1):
            w = w * (r[i - 1] if bit(z, i) else (1 - r[i - 1])) % P
        return w
    assert [sum(weight(z, m) * entry(y, z) for z in range(1 << m)) % P for y in range(Ny)] == T
    C = [sum(entry(y, z) for y in range(Ny)) % P for z in range(1 << m)]
    for i in range(1, m + 1):
        g0 = sum(weight(z, i - 1) * C[z] for z in range(1 << m) if bit(z, i) == 0) % P
        g1 = sum(weight(z, i - 1) * C[z] for z in range(1 << m) if bit(z, i) == 1) % P
        assert (g0, g1) == sums[i - 1], i
