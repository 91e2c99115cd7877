"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Every output -- round polynomials g_i(0..d), challenges r_i, final evaluations f_m(rho) and the
claim H -- is integer data (exact F_p arithmetic), so the bar is bit-exact equality.
"""
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

SEED = inputs.DEFAULT_SEED
KEYS = ("round_evals", "challenges", "final_evals", "claims")


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def dev_tables(B, d, k, first_index=0, dist="uniform"):
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, first_index, dist)
    return t


@pytest.fixture(scope="module")
def prover():
    p = bzk.Prover(0)
    yield p
    p.close()


def check_against_oracle(orc, tables_np, out, k, d, order, first_index, idx=None):
    B = tables_np.shape[0]
    idx = range(B) if idx is None else idx
    sub = np.ascontiguousarray(tables_np[list(idx)])
    for n, b in enumerate(idx):
        ref = orc.prove(sub[n], k, d, order, SEED, first_index + b)
        for key in KEYS:
            got = np64(out[key][b]) if key != "claims" else np64(out[key][b])
            assert np.array_equal(got.reshape(ref[key].shape), ref[key]), (key, b, k, d, order)


def test_generator_matches_host_twin():
    for (B, d, k, I, dist) in [(3, 2, 5, 0, "uniform"), (2, 3, 7, 1000, "smallint"), (2, 2, 4, 5, "vml"),
                               (1, 1, 0, 7, "uniform")]:
        t = dev_tables(B, d, k, I, dist)
        assert np.array_equal(np64(t), inputs.gen_tables(B, d, k, I, dist))


def test_field_ops_vs_oracle(orc):
    rng = np.random.default_rng(11)
    P = orc.P
    n = 1 << 16
    edge = [0, 1, 2, P - 1, P - 2, 2**253, (2**256) % P, P // 2, 0xFFFFFFFF, 2**64 - 1]
    av = [int(x) for x in rng.integers(0, 2**63, size=n)] + edge * len(edge)
    bv = [int(x) for x in rng.integers(0, 2**63, size=n)] + [e for e in edge for _ in edge]
    # widen to full 254-bit values
    av = [(x * 0x9E3779B97F4A7C15 ** 3) % P for x in av[:n]] + av[n:]
    bv = [(x * 0xC2B2AE3D27D4EB4F ** 3) % P for x in bv[:n]] + bv[n:]
    A = torch.from_numpy(orc.to_limbs(av).view(np.int64)).cuda()
    Bt = torch.from_numpy(orc.to_limbs(bv).view(np.int64)).cuda()
    out = torch.empty_like(A)
    Rinv = pow(2**256, P - 2, P)
    for op, fn in [(0, lambda x, y: (x + y) % P), (1, lambda x, y: (x - y) % P),
                   (2, lambda x, y: x * y * Rinv % P), (3, lambda x, y: x * y % P)]:
        bzk.bzk_debug_field(op, A.shape[0], A, Bt, out)
        torch.cuda.synchronize()
        got = orc.from_limbs(np64(out))
        assert got == [fn(x, y) for x, y in zip(av, bv)], op
    # reduce256: arbitrary 256-bit inputs
    raw = [int.from_bytes(rng.bytes(32), "little") for _ in range(4096)] + [2**256 - 1, 5 * P, P, 0]
    R = torch.from_numpy(orc.to_limbs(raw).view(np.int64)).cuda()
    out = torch.empty_like(R)
    bzk.bzk_debug_field(4, R.shape[0], R, None, out)
    torch.cuda.synchronize()
    assert orc.from_limbs(np64(out)) == [x % P for x in raw]


def test_device_sha256_vs_hashlib():
    import hashlib
    rng = np.random.default_rng(5)
    for L in list(range(0, 200, 4)) + [56, 60, 64, 120, 124, 128, 132]:
        n = 8
        msgs = rng.integers(0, 256, size=(n, max(L, 1)), dtype=np.uint8)[:, :L].copy()
        d_m = torch.from_numpy(msgs.reshape(-1)).cuda() if L else torch.zeros(1, dtype=torch.uint8, device="cuda")
        d_o = torch.empty((n, 32), dtype=torch.uint8, device="cuda")
        bzk.bzk_debug_sha256(d_m, L, n, d_o)
        torch.cuda.synchronize()
        o = d_o.cpu().numpy()
        for i in range(n):
            assert bytes(o[i]) == hashlib.sha256(bytes(msgs[i])).digest(), L


# ---------------------------------------------------------------- small configs, every proof

@pytest.mark.parametrize("order", [0, 1])
def test_config1_all_proofs(prover, orc, order):
    """configs[0]: B=16, d=2, k=12 -- every proof, every output, bit-exact."""
    B, d, k = 16, 2, 12
    t = dev_tables(B, d, k)
    out = prover.prove(t, k, d, order, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    check_against_oracle(orc, np64(t), out, k, d, order, 0)


SWEEP = [(d, k) for d in (1, 2, 3, 4) for k in (0, 1, 2, 3, 5, 8, 9, 10, 11, 12, 13)]


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d,k", SWEEP)
def test_sweep_degrees_and_sizes(prover, orc, d, k, order):
    B = 3 if k <= 11 else 2
    I = 100 + k
    t = dev_tables(B, d, k, I)
    out = prover.prove(t, k, d, order, first_index=I)
    torch.cuda.synchronize()
    check_against_oracle(orc, inputs.gen_tables(B, d, k, I), out, k, d, order, I)


@pytest.mark.parametrize("k", [14, 16])
def test_larger_k_many_ctas(prover, orc, k):
    """Several CTAs per proof (last-CTA ticket path) and several fused rounds."""
    B, d = 5, 2
    t = dev_tables(B, d, k, 3)
    out = prover.prove(t, k, d, 0, first_index=3, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    check_against_oracle(orc, np64(t), out, k, d, 0, 3)


def test_smallint_and_vml_distributions(prover, orc):
    for dist in ("smallint", "vml"):
        t = dev_tables(3, 2, 11, 9, dist)
        out = prover.prove(t, 11, 2, 0, first_index=9)
        torch.cuda.synchronize()
        check_against_oracle(orc, inputs.gen_tables(3, 2, 11, 9, dist), out, 11, 2, 0, 9)


def test_constant_and_zero_tables(prover, orc):
    k, d = 10, 3
    t = torch.zeros((2, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    t[1, :, :, 0] = 7          # constant tables
    out = prover.prove(t, k, d, 0)
    torch.cuda.synchronize()
    check_against_oracle(orc, np64(t), out, k, d, 0, 0)
    P = orc.P
    g = orc.from_limbs(np64(out["round_evals"][1]))
    assert g[0] == (1 << (k - 1)) * 343 % P


# ---------------------------------------------------------------- API semantics

def test_preserve_vs_consume_and_wave_independence(orc):
    B, d, k = 6, 2, 14
    t = dev_tables(B, d, k)
    ref_tab = t.clone()
    p_big = bzk.Prover(0)
    out1 = p_big.prove(t, k, d, 0, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    assert torch.equal(t, ref_tab)
    # a tiny workspace limit forces one proof per wave
    p_small = bzk.Prover(0, workspace_limit=3 * (1 << 20))
    out2 = p_small.prove(t.clone(), k, d, 0)         # consume mode
    torch.cuda.synchronize()
    for key in KEYS:
        assert torch.equal(out1[key], out2[key]), key
    p_big.close()
    p_small.close()


def test_sharding_by_first_index(prover):
    B, d, k = 8, 2, 13
    t = dev_tables(B, d, k)
    full = prover.prove(t, k, d, 0, flags=bzk.BZK_F_PRESERVE_INPUT)
    lo = prover.prove(t[:3].contiguous(), k, d, 0, first_index=0)
    hi = prover.prove(t[3:].contiguous(), k, d, 0, first_index=3)
    torch.cuda.synchronize()
    for key in KEYS:
        assert torch.equal(full[key], torch.cat([lo[key], hi[key]])), key


def test_host_tables_and_host_outputs(prover):
    B, d, k = 5, 2, 15
    t = dev_tables(B, d, k)
    dev = prover.prove(t, k, d, 1, flags=bzk.BZK_F_PRESERVE_INPUT)
    host_t = t.cpu().pin_memory()
    out_h = bzk.Prover.alloc_outputs(B, k, d, device="cpu", pin=True)
    p = bzk.Prover(0, workspace_limit=2 * 2 * (1 << k) * 32 * 4)   # forces several loader waves
    p.prove(host_t, k, d, 1, out=out_h)
    torch.cuda.synchronize()
    for key in KEYS:
        assert torch.equal(dev[key].cpu(), out_h[key]), key
    p.close()


def test_ragged_jobs(prover, orc):
    jobs, outs, tabs = [], [], []
    shapes = [(2, 2, 12, 0), (3, 1, 9, 50), (1, 3, 14, 60), (2, 2, 0, 70), (2, 4, 5, 80)]
    for (B, d, k, I) in shapes:
        t = dev_tables(B, d, k, I)
        o = bzk.Prover.alloc_outputs(B, k, d)
        tabs.append(t)
        outs.append(o)
        jobs.append(prover.batch(t, k, d, 0, None, I, 0, o))
        prover._keep = getattr(prover, "_keep", []) + prover._seed_bufs
    bzk.bzk_prove_ragged(prover.ctx, jobs)
    torch.cuda.synchronize()
    for (B, d, k, I), o in zip(shapes, outs):
        check_against_oracle(orc, inputs.gen_tables(B, d, k, I), o, k, d, 0, I)


def test_validate_flag_rejects_noncanonical(prover, orc):
    B, d, k = 2, 2, 10
    t = dev_tables(B, d, k)
    t[1, 1, 77] = torch.from_numpy(orc.to_limbs([orc.P]).view(np.int64)[0])
    with pytest.raises(bzk.BzkError) as e:
        prover.prove(t, k, d, 0, flags=bzk.BZK_F_VALIDATE)
    assert e.value.status == bzk.BZK_ENONCANON
    t[1, 1, 77] = 0
    prover.prove(t, k, d, 0, flags=bzk.BZK_F_VALIDATE | bzk.BZK_F_SYNC)


def test_argument_errors(prover):
    t = dev_tables(1, 2, 4)
    for kw in [dict(k=31), dict(d=0), dict(order=2)]:
        k, d, order = kw.get("k", 4), kw.get("d", 2), kw.get("order", 0)
        out = bzk.Prover.alloc_outputs(1, min(k, 4), max(min(d, 4), 1))
        b = prover.batch(t, k, d, order, None, 0, 0, out)
        with pytest.raises(bzk.BzkError) as e:
            bzk.bzk_prove(prover.ctx, b)
        assert e.value.status == bzk.BZK_EINVAL
    out = bzk.Prover.alloc_outputs(1, 4, 4)
    b = prover.batch(t, 4, 5, 0, None, 0, 0, out)           # well defined, not built
    with pytest.raises(bzk.BzkError) as e:
        bzk.bzk_prove(prover.ctx, b)
    assert e.value.status == bzk.BZK_EUNSUPPORTED
    out = bzk.Prover.alloc_outputs(1, 4, 2)
    b = prover.batch(t, 4, 2, 0, None, 0, 0, out, batch=0)
    with pytest.raises(bzk.BzkError):
        bzk.bzk_prove(prover.ctx, b)
    b = prover.batch(t, 4, 2, 0, None, 0, 0, out)
    b.tables = None
    with pytest.raises(bzk.BzkError):
        bzk.bzk_prove(prover.ctx, b)


def test_outputs_verify_with_reference_verifier(prover, orc):
    B, d, k = 4, 3, 13
    t = dev_tables(B, d, k, 40)
    out = prover.prove(t, k, d, 1, first_index=40)
    torch.cuda.synchronize()
    for b in range(B):
        assert orc.verify(k, d, 1, SEED, 40 + b, np64(out["round_evals"][b]), np64(out["challenges"][b]),
                          np64(out["final_evals"][b]), np64(out["claims"][b])) == 0


def test_cuda_graph_replay_and_recapture(prover):
    B, d, k = 4, 2, 14
    t = dev_tables(B, d, k)
    ref = prover.prove(t, k, d, 0, flags=bzk.BZK_F_PRESERVE_INPUT)
    out = bzk.Prover.alloc_outputs(B, k, d)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    b = prover.batch(t, k, d, 0, None, 0, bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_GRAPH, out)
    for rep in range(3):                       # capture, then replays
        with torch.cuda.stream(s):
            for key in out:
                out[key].zero_()
        bzk.bzk_prove(prover.ctx, b, s)
        s.synchronize()
        for key in ref:
            assert torch.equal(out[key], ref[key]), (rep, key)
    # a different seed must not replay the old graph
    seed2 = bytes([7]) + bytes(range(1, 32))
    b2 = prover.batch(t, k, d, 0, seed2, 0, bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_GRAPH, out)
    bzk.bzk_prove(prover.ctx, b2, s)
    s.synchronize()
    ref2 = prover.prove(t, k, d, 0, seed=seed2, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    for key in ref2:
        assert torch.equal(out[key], ref2[key]), key
    assert not torch.equal(ref2["challenges"], ref["challenges"])


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d,k", [(1, 12), (2, 13), (3, 10), (1, 16), (2, 4)])
def test_given_challenges_paper_literal(prover, orc, d, k, order):
    """BZK_F_GIVEN_CHALLENGES (Alg. 1: r_i are inputs) vs the oracle's given-challenge mode;
    d = 1, MSB is Algorithm 1 literally."""
    B = 3
    t = dev_tables(B, d, k, 30)
    rng = np.random.default_rng(k)
    P = orc.P
    r_int = [[int(x) * 0x9E3779B97F4A7C15 % P for x in rng.integers(1, 2**62, size=k)] for _ in range(B)]
    r = np.stack([orc.to_limbs(rr) for rr in r_int])
    out = bzk.Prover.alloc_outputs(B, k, d)
    out["challenges"].copy_(torch.from_numpy(r.view(np.int64)))
    b = prover.batch(t, k, d, order, None, 30, bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_GIVEN_CHALLENGES, out)
    bzk.bzk_prove(prover.ctx, b)
    torch.cuda.synchronize()
    host = np64(t)
    for i in range(B):
        ref = orc.prove_given(host[i], k, d, order, r[i])
        for key in KEYS:
            assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), (key, i)
        if d == 1 and order == 1:
            assert np.array_equal(orc.alg1(host[i][0], r[i]), np64(out["round_evals"][i]).reshape(k, 2, 4))


def test_fp64_pipe_montgomery_vs_oracle(orc):
    """field_f64.cuh: radix-2^48 FP64 Montgomery products (R' = 2^288) on random and edge inputs up
    to 2^256 - 1 (the lazy representation)."""
    rng = np.random.default_rng(17)
    P = orc.P
    n = 1 << 15
    edge = [0, 1, P - 1, P, 2 * P - 1, 2**256 - 1, 2**255, 2**48 - 1, 2**48, 2**253]
    av = [int.from_bytes(rng.bytes(32), "little") for _ in range(n)] + [e for e in edge for _ in edge]
    bv = [int.from_bytes(rng.bytes(32), "little") for _ in range(n)] + edge * len(edge)
    A = torch.from_numpy(orc.to_limbs(av).view(np.int64)).cuda()
    Bt = torch.from_numpy(orc.to_limbs(bv).view(np.int64)).cuda()
    out = torch.empty_like(A)
    inv = pow(2**288, P - 2, P)
    for op, f in [(5, 1), (6, 2)]:
        bzk.bzk_debug_field(op, A.shape[0], A, Bt, out)
        torch.cuda.synchronize()
        assert orc.from_limbs(np64(out)) == [f * x * y * inv % P for x, y in zip(av, bv)], op
