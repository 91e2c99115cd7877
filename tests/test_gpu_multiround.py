"""NEXT-1: the paper-literal sum-check with KNOWN challenges (Alg. 1; r_i PRG-seeded),
several rounds per read of the table (csrc/multiround.cuh: k_multi passes, then the on-chip tail).

Bit-exact against the oracle's given-challenge prover and, for MSB order, against Algorithm 1 run
literally ((1 - r) A[b] + r A[b + h], oracle.alg1).  k covers: no pass (k <= 9), one pass of 1, 2 and
3 rounds (k = 10, 11, 12), several passes with a short last one (13, 14, 15, 16, 19) and the bench
shape k = 20 at full size (1024 proofs, m0lit) on sampled proofs.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

KEYS = ("round_evals", "challenges", "final_evals", "claims")
P = int.from_bytes(b"".join(x.to_bytes(8, "little") for x in inputs.P_BN254), "little")


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def challenges(orc, B, k, seed, edge=False):
    rng = np.random.default_rng(seed)
    rs = []
    for b in range(B):
        r = [int.from_bytes(rng.bytes(32), "little") % P for _ in range(k)]
        if edge:     # r = 0, 1, p - 1 bind a variable to a hypercube point / its "negative"
            for i in range(k):
                r[i] = [0, 1, P - 1, r[i]][(i + b) % 4]
        rs.append(orc.to_limbs(r))
    return np.stack(rs)


def run(prover, t, k, order, r, first_index=0, flags=0):
    B = t.shape[0]
    out = bzk.Prover.alloc_outputs(B, k, 1)
    out["challenges"].copy_(torch.from_numpy(r.view(np.int64)))
    b = prover.batch(t, k, 1, order, None, first_index, flags | bzk.BZK_F_GIVEN_CHALLENGES, out)
    bzk.bzk_prove(prover.ctx, b)
    torch.cuda.synchronize()
    return out


@pytest.fixture(scope="module")
def prover():
    p = bzk.Prover(0)
    yield p
    p.close()


@pytest.mark.parametrize("dist", ["uniform", "adversarial"])
@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("k", [3, 9, 10, 11, 12, 13, 14, 15, 16, 19])
def test_multiround_vs_oracle(prover, orc, k, order, dist):
    B = 4 if k <= 16 else 2
    I = 300 + k
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, I, dist)
    r = challenges(orc, B, k, k, edge=(dist == "adversarial"))
    out = run(prover, t, k, order, r, first_index=I, flags=bzk.BZK_F_PRESERVE_INPUT)
    host = np64(t)
    for b in range(B):
        ref = orc.prove_given(host[b], k, 1, order, r[b])
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)
        if order == 1:
            assert np.array_equal(orc.alg1(host[b][0], r[b]), np64(out["round_evals"][b]).reshape(k, 2, 4))


def test_multiround_consume_and_waves(orc):
    """consume mode (the LSB second scratch buffer aliases the dead input) and one-proof waves"""
    k, B = 15, 5
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 0, "uniform")
    host = np64(t).copy()
    r = challenges(orc, B, k, 99)
    for order in (0, 1):
        p = bzk.Prover(0, workspace_limit=3 * (1 << 20))
        out = run(p, t.clone(), k, order, r)
        p.close()
        for b in range(B):
            ref = orc.prove_given(host[b], k, 1, order, r[b])
            for key in KEYS:
                assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, order)


def test_multiround_host_tables(orc):
    k, B = 14, 4
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 0, "uniform")
    host_t = t.cpu().pin_memory()
    r = challenges(orc, B, k, 5)
    out = bzk.Prover.alloc_outputs(B, k, 1, device="cpu", pin=True)
    out["challenges"].copy_(torch.from_numpy(r.view(np.int64)))
    p = bzk.Prover(0)
    b = p.batch(host_t, k, 1, 1, None, 0, bzk.BZK_F_GIVEN_CHALLENGES, out)
    bzk.bzk_prove(p.ctx, b)
    p.close()
    for i in range(B):
        ref = orc.prove_given(np64(host_t)[i], k, 1, 1, r[i])
        for key in KEYS:
            assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), (key, i)


def test_m0lit_full_size(orc):
    """bench.py --config m0lit's call: 1024 proofs x d = 1, k = 20, MSB, challenges given, PRESERVE."""
    B, k = 1024, 20
    torch.cuda.empty_cache()
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 0, "uniform")
    r = challenges(orc, B, k, 2020)
    p = bzk.Prover(0)
    out = run(p, t, k, 1, r, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.close()
    del t
    torch.cuda.empty_cache()
    rng = np.random.default_rng(20)
    for i in sorted({0, B - 1, *rng.choice(B, size=3, replace=False).tolist()}):
        tab = inputs.gen_tables(1, 1, k, first_index=i)[0]
        ref = orc.prove_given(tab, k, 1, 1, r[i])
        for key in KEYS:
            assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), (key, i)
    # round invariant on every proof: g_i(0) + g_i(1) = g_{i-1}(r_{i-1}) (d = 1: linear interpolation)
    ev = np64(out["round_evals"]).reshape(B, k, 2, 4)
    for i in range(0, B, 97):
        g = [[orc.from_limbs(ev[i, j, t])[0] for t in range(2)] for j in range(k)]
        rr = orc.from_limbs(r[i])
        for j in range(1, k):
            prev = (g[j - 1][0] + rr[j - 1] * (g[j - 1][1] - g[j - 1][0])) % P
            assert (g[j][0] + g[j][1]) % P == prev, (i, j)


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("k,B", [(16, 1), (16, 3), (17, 2)])
def test_multiround_tc_extremes(orc, order, k, B):
    """k_multi_tc (tensor-core passes, csrc/multiround_tc.cuh) at the byte extremes: every entry p - 1
    (all bytes near 255, the largest column values c_n and column byte sums), alternating 0 / p - 1,
    and r in {0, 1, p - 1}; the profile shows the tensor-core kernel ran (k >= 16: too large for k_small)."""
    N = 1 << k
    pm1 = np.array(inputs.P_BN254, dtype=np.uint64).copy()
    pm1[0] -= 1
    host = np.zeros((B, 1, N, 4), dtype=np.uint64)
    host[0, 0, :] = pm1
    if B > 1:
        host[1, 0, 1::2] = pm1
    if B > 2:
        host[2, 0, :] = inputs.gen_tables(1, 1, k, first_index=77, dist="adversarial")[0, 0]
    t = torch.from_numpy(host.view(np.int64)).cuda()
    r = challenges(orc, B, k, 31 + k, edge=True)
    p = bzk.Prover(0)
    bzk.bzk_profile_enable(p.ctx, 1)
    out = run(p, t, k, order, r, flags=bzk.BZK_F_PRESERVE_INPUT)
    prof = bzk.bzk_profile_read(p.ctx, 1)
    p.close()
    assert prof["multi_round_tc"][1] > 0, prof
    for b in range(B):
        ref = orc.prove_given(host[b], k, 1, order, r[b])
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)


TC_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r}); sys.path.insert(0, {root!r} + "/tests")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk
from test_gpu_multiround import challenges, run, np64, KEYS
oracle.build()
for k, B, order in [(16, 2, 0), (16, 1, 1), (17, 1, 0)]:
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 500 + k, "adversarial")
    r = challenges(oracle, B, k, 7 * k)
    p = bzk.Prover(0)
    out = run(p, t, k, order, r, first_index=500 + k, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.close()
    host = np64(t)
    for b in range(B):
        ref = oracle.prove_given(host[b], k, 1, order, r[b])
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, k, order)
print("tc ok")
"""


@pytest.mark.parametrize("env", [{"BZK_TC_CTAS": "1"}, {"BZK_TC_CTAS": "7"}, {"BZK_TC_CTAS": "1000"},
                                 {"BZK_MULTI_TC": "0"}, {"BZK_MULTI_M": "1"}, {"BZK_MULTI_M": "2"}])
def test_multiround_tc_launch_shapes(env):
    """k_multi_tc with one CTA per proof, 7 CTAs (ragged: 64 tiles -> 10 / 9 per CTA, last-CTA ticket), one
    CTA per tile, and the CUDA-core k_multi instead (BZK_MULTI_TC=0); passes of 1 and 2 rounds (BZK_MULTI_M, the
    CUDA-core k_multi: k_multi_tc takes 3-round passes only); k_small off so every case runs the passes."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", TC_SCRIPT.format(root=root)], env=dict(os.environ, BZK_SMALL="0", **env),
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "tc ok" in r.stdout, r.stdout + r.stderr
