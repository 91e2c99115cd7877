"""GPU tests of the scheduler / boundary semantics (round-2 fixes), bit-exact against the oracle.

* CTA-partials sizing over every global round (ctas_for is not monotone in h): the shapes where
  round 1's CTA count is smaller than a later round's (k=16, B=64 and k=19, B=4, d=2).
* a cached CUDA graph is dropped when the workspace moves (capture -> bigger call -> replay).
* calls on one context issued on different streams are ordered (shared workspace).
* bzk_workspace_size == what a fresh context allocates (device and host tables).
* u64 first_index (the transcript absorbs LE64 I; no 2^28 cap on the prover).
* thread-block-cluster (DSMEM) reduction of the CTA partials (BZK_CLUSTER, a separate process).
"""
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SEED = inputs.DEFAULT_SEED
KEYS = ("round_evals", "challenges", "final_evals", "claims")


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def dev_tables(B, d, k, first_index=0, dist="uniform"):
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, first_index, dist)
    return t


def check(orc, host, out, k, d, order, first_index, idx):
    for b in idx:
        ref = orc.prove(host[b], k, d, order, SEED, first_index + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)


@pytest.fixture(scope="module")
def prover():
    p = bzk.Prover(0)
    yield p
    p.close()


def _ctas_for(h, nb, ppt_max=256, waves=4):
    """api.cu ctas_for (default knobs), to find the shapes where later rounds use more CTAs."""
    target = 148 * 2 * waves
    ppt = max(1, min(ppt_max, (nb * h) // (256 * target)))
    c = max(1, (h + 256 * ppt - 1) // (256 * ppt))
    if c >= 8:
        return (c + 7) // 8 * 8
    q = 1
    while q < c:
        q <<= 1
    return q


@pytest.mark.parametrize("B,k", [(64, 16), (4, 19)])
def test_partials_sized_over_all_rounds(prover, orc, B, k):
    d = 2
    c1 = _ctas_for(1 << (k - 1), B)
    cmax = max(_ctas_for(1 << (k - i), B) for i in range(1, k - 8))
    assert cmax > c1, "shape no longer exercises a later round with more CTAs than round 1"
    t = dev_tables(B, d, k, 11)
    out = prover.prove(t, k, d, 0, first_index=11, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    check(orc, host, out, k, d, 0, 11, [0, B // 2, B - 1])
    # every proof of the batch is accepted by the reference verifier
    for b in range(B):
        assert orc.verify(k, d, 0, SEED, 11 + b, np64(out["round_evals"][b]), np64(out["challenges"][b]),
                          np64(out["final_evals"][b]), np64(out["claims"][b])) == 0, b


def test_graph_dropped_when_workspace_moves(orc):
    p = bzk.Prover(0)
    B, d, k = 3, 2, 13
    t = dev_tables(B, d, k, 5)
    out = bzk.Prover.alloc_outputs(B, k, d)
    torch.cuda.synchronize()
    s = torch.cuda.Stream()
    b = p.batch(t, k, d, 0, None, 5, bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_GRAPH, out)
    bzk.bzk_prove(p.ctx, b, s)                       # capture (small workspace)
    s.synchronize()
    # a much larger call reallocates the workspace (the old one is freed)
    big = dev_tables(2, 2, 18, 100)
    p.prove(big, 18, 2, 0, first_index=100)
    torch.cuda.synchronize()
    # and a Merkle batch on the same context
    blocks = torch.empty((4, 1 << 12, 64), dtype=torch.uint8, device="cuda")
    bzk.bzk_generate_blocks(blocks, 4, 12, 0)
    bzk.MerkleBuilder(0, ctx=p.ctx).build(blocks, 12)
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for key in out:
            out[key].zero_()
    b = p.batch(t, k, d, 0, None, 5, bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_GRAPH, out)
    bzk.bzk_prove(p.ctx, b, s)                       # same description: re-captured, not replayed stale
    s.synchronize()
    check(orc, np64(t), out, k, d, 0, 5, range(B))
    p.close()


def test_calls_on_different_streams_are_ordered(orc):
    """Two calls on one context, on two streams, back to back with no host sync: the second must
    not overwrite the first's workspace while it runs."""
    p = bzk.Prover(0)
    B, d, k = 8, 2, 16
    t1 = dev_tables(B, d, k, 0)
    t2 = dev_tables(B, d, k, 500)
    o1 = bzk.Prover.alloc_outputs(B, k, d)
    o2 = bzk.Prover.alloc_outputs(B, k, d)
    torch.cuda.synchronize()
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    for _ in range(3):
        p.prove(t1, k, d, 0, first_index=0, flags=bzk.BZK_F_PRESERVE_INPUT, out=o1, stream=s1)
        p.prove(t2, k, d, 0, first_index=500, flags=bzk.BZK_F_PRESERVE_INPUT, out=o2, stream=s2)
    torch.cuda.synchronize()
    check(orc, np64(t1), o1, k, d, 0, 0, [0, B - 1])
    check(orc, np64(t2), o2, k, d, 0, 500, [0, B - 1])
    p.close()


@pytest.mark.parametrize("host", [False, True])
def test_workspace_size_matches_allocation(host):
    B, d, k = 16, 2, 16
    t = dev_tables(B, d, k, 0)
    if host:
        t = t.cpu().pin_memory()
    out = bzk.Prover.alloc_outputs(B, k, d, device="cpu" if host else "cuda", pin=host)
    torch.cuda.synchronize()
    p = bzk.Prover(0, workspace_limit=6 * B * d * (1 << k) * 32)
    b = p.batch(t, k, d, 0, None, 0, bzk.BZK_F_PRESERVE_INPUT, out)
    need = bzk.bzk_workspace_size(p.ctx, b)
    torch.cuda.synchronize()
    free0, _ = torch.cuda.mem_get_info()
    bzk.bzk_prove(p.ctx, b)
    bzk.bzk_sync(p.ctx)
    free1, _ = torch.cuda.mem_get_info()
    used = free0 - free1
    assert need <= used <= need + 8 * (2 << 20), (need, used)   # allocation granularity: 2 MiB pages
    if host:
        assert need > 2 * B * d * (1 << k) * 32 // 8      # staging slots are included
    p.close()


def test_large_first_index(prover, orc):
    """first_index is a u64 bound into the transcript (LE64 I); > 2^28 and > 2^32 work."""
    B, d, k = 3, 2, 11
    t = dev_tables(B, d, k, 0)
    host = np64(t)
    for I in (1 << 28, (1 << 40) + 12345, (1 << 64) - B):
        out = prover.prove(t, k, d, 1, first_index=I, flags=bzk.BZK_F_PRESERVE_INPUT)
        torch.cuda.synchronize()
        check(orc, host, out, k, d, 1, I, range(B))
    out = bzk.Prover.alloc_outputs(B, k, d)
    b = prover.batch(t, k, d, 0, None, (1 << 64) - 2, 0, out)
    with pytest.raises(bzk.BzkError) as e:           # first_index + batch overflows
        bzk.bzk_prove(prover.ctx, b)
    assert e.value.status == bzk.BZK_EINVAL


CLUSTER_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
oracle.build()
p = bzk.Prover(0)
for (B, d, k, order) in [(3, 2, 16, 0), (2, 3, 15, 1), (2, 1, 17, 0), (5, 4, 14, 1)]:
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 7, "adversarial")
    out = p.prove(t, k, d, order, first_index=7, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = t.cpu().numpy().view(np.uint64)
    for b in range(B):
        ref = oracle.prove(host[b], k, d, order, inputs.DEFAULT_SEED, 7 + b)
        for key in ref:
            got = out[key][b].cpu().numpy().view(np.uint64).reshape(ref[key].shape)
            assert np.array_equal(got, ref[key]), (key, B, d, k, order, b)
p.close()
print("cluster ok")
"""


@pytest.mark.parametrize("cluster", [2, 8])
def test_cluster_dsmem_reduction(cluster):
    env = dict(os.environ, BZK_CLUSTER=str(cluster))
    r = subprocess.run([sys.executable, "-c", CLUSTER_SCRIPT.format(root=ROOT)], env=env, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "cluster ok" in r.stdout, r.stdout + r.stderr


PERROUND_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
oracle.build()
p = bzk.Prover(0)
n = 0
for d in (1, 2, 3, 4):
    for k in (1, 2, 5, 9, 10, 11, 13):
        for order in (0, 1):
            B = 3
            t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
            bzk.bzk_generate(t, B, d, k, 50 + k, "adversarial")
            out = p.prove(t, k, d, order, first_index=50 + k, flags=bzk.BZK_F_PRESERVE_INPUT)
            torch.cuda.synchronize()
            host = t.cpu().numpy().view(np.uint64)
            for b in range(B):
                ref = oracle.prove(host[b], k, d, order, inputs.DEFAULT_SEED, 50 + k + b)
                for key in ref:
                    got = out[key][b].cpu().numpy().view(np.uint64).reshape(ref[key].shape)
                    assert np.array_equal(got, ref[key]), (key, d, k, order, b)
                n += 1
p.close()
print("per-round ok", n)
"""


def test_per_round_path_at_small_k():
    """With BZK_SMALL=0 the shapes k_small would take run through the per-round kernels + on-chip
    tail (round 1, fused rounds, tail-only and first-tail-round-2 cases) -- both paths stay tested."""
    env = dict(os.environ, BZK_SMALL="0")
    r = subprocess.run([sys.executable, "-c", PERROUND_SCRIPT.format(root=ROOT)], env=env, capture_output=True,
                       text=True, timeout=900)
    assert r.returncode == 0 and "per-round ok" in r.stdout, r.stdout + r.stderr


DUAL_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
oracle.build()
p = bzk.Prover(0)
for (B, d, k, order, flags) in [(6, 2, 14, 0, bzk.BZK_F_PRESERVE_INPUT), (5, 3, 13, 1, 0), (4, 1, 15, 1, 0),
                                (3, 4, 12, 0, bzk.BZK_F_PRESERVE_INPUT), (2, 2, 16, 1, 0)]:
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 21, "adversarial")
    host = t.cpu().numpy().view(np.uint64).copy()
    out = p.prove(t, k, d, order, first_index=21, flags=flags)
    torch.cuda.synchronize()
    for b in range(B):
        ref = oracle.prove(host[b], k, d, order, inputs.DEFAULT_SEED, 21 + b)
        for key in ref:
            got = out[key][b].cpu().numpy().view(np.uint64).reshape(ref[key].shape)
            assert np.array_equal(got, ref[key]), (key, B, d, k, order, b)
p.close()
print("dual ok")
"""


def test_dual_stream_waves():
    """BZK_DUAL=1: a one-wave batch runs as two half waves on two streams, the second one round behind
    (measured no faster on B200 -- profiles/r02/bench_*_dual*_r02p.json -- so off by default)."""
    env = dict(os.environ, BZK_DUAL="1")
    r = subprocess.run([sys.executable, "-c", DUAL_SCRIPT.format(root=ROOT)], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0 and "dual ok" in r.stdout, r.stdout + r.stderr


@pytest.mark.parametrize("gl", [False, True])
def test_per_proof_device_seeds(prover, orc, gl):
    """BZK_F_SEEDS_DEVICE: proof b's transcript starts from its own 32-byte seed (device [B][32]);
    BN254 through both execution paths (k_small at k = 11, per-round kernels at k = 15) and Goldilocks."""
    d, order = 2, 1
    for k, B in ((11, 3), (15, 3)):
        seeds = np.stack([np.frombuffer(bytes((7 * b + i) & 0xFF for i in range(32)), np.uint8) for b in range(B)])
        sd = torch.from_numpy(seeds.copy()).cuda()
        if gl:
            t = torch.empty((B, d, 1 << k), dtype=torch.int64, device="cuda")
            bzk.bzk_generate(t, B, d, k, 40, "gl_adversarial")
            out = bzk.Prover.alloc_outputs_gl(B, k, d)
            flags = bzk.BZK_F_FIELD_GOLDILOCKS
        else:
            t = dev_tables(B, d, k, 40, "adversarial")
            out = bzk.Prover.alloc_outputs(B, k, d)
            flags = 0
        b = bzk.make_batch(k, d, order, flags | bzk.BZK_F_SEEDS_DEVICE | bzk.BZK_F_PRESERVE_INPUT, B, 40, sd.data_ptr(),
                           t, bzk.BZK_MEM_DEVICE, bzk.BZK_MEM_DEVICE, out["round_evals"], out["challenges"],
                           out["final_evals"], out["claims"])
        bzk.bzk_prove(prover.ctx, b)
        torch.cuda.synchronize()
        host = np64(t)
        for i in range(B):
            if gl:
                ref = orc.gl_prove(host[i], k, d, order, seeds[i].tobytes(), 40 + i)
            else:
                ref = orc.prove(host[i], k, d, order, seeds[i].tobytes(), 40 + i)
            for key in KEYS:
                assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), (key, i, k)


@pytest.mark.parametrize("order", [0, 1])
def test_single_large_proof(prover, orc, order):
    """One proof with k = 22 (d = 2, 256 MiB of tables): many CTAs per proof in every global round
    (the ticket reduction over hundreds of partials), full-field tables, against the oracle."""
    k, d = 22, 2
    t = dev_tables(1, d, k, 77)
    out = prover.prove(t, k, d, order, first_index=77, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    check(orc, np64(t), out, k, d, order, 77, [0])
