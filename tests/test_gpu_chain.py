"""GPU parity of the section-4 chain (bzk_commit_prove, R25): per proof,
S message segments are encoded, each codeword committed with a Merkle tree, the roots combined by a
root-of-roots tree, and the sum-check transcript seeded with that final root -- every output
bit-exact against oracle.commit_prove (itself pinned in tests/test_oracle_chain.py)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

KEYS = ("round_evals", "challenges", "final_evals", "claims")


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def run_chain(enc, log_n, S, B, d, k, order, mode, I0, dist="uniform", nodes=False):
    n = 1 << log_n
    msgs = inputs.gen_tables(B * S, 1, log_n, first_index=I0 + 1000)[:, 0]
    codes = torch.zeros((B, S, 2 * n, 4), dtype=torch.int64, device="cuda")
    codes[:, :, :n] = torch.from_numpy(msgs.view(np.int64).reshape(B, S, n, 4)).cuda()
    roots = torch.empty((B, S, 32), dtype=torch.uint8, device="cuda")
    fin = torch.empty((B, 32), dtype=torch.uint8, device="cuda")
    nd = torch.empty((B, S, 2 * n - 1, 32), dtype=torch.uint8, device="cuda") if nodes else None
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, I0, dist)
    out = bzk.Prover.alloc_outputs(B, k, d)
    p = enc  # Encoder owns the context
    c = bzk.bzk_commit(S, mode, codes.data_ptr(), roots.data_ptr(), nd.data_ptr() if nodes else None, fin.data_ptr())
    sb = bzk.make_batch(k, d, order, bzk.BZK_F_PRESERVE_INPUT, B, I0, None, t, bzk.BZK_MEM_DEVICE,
                        bzk.BZK_MEM_DEVICE, out["round_evals"], out["challenges"], out["final_evals"], out["claims"])
    bzk.bzk_commit_prove(p.ctx, p.enc, c, sb)
    torch.cuda.synchronize()
    return msgs.reshape(B, S, n, 4), codes, roots, fin, nd, t, out


@pytest.mark.parametrize("S,mode,order,d,B", [(1, 0, 0, 2, 3), (2, 0, 1, 1, 2), (4, 1, 0, 3, 3), (8, 0, 0, 2, 3),
                                              (2, 0, 0, 2, 1), (2, 1, 1, 2, 5)])
def test_chain_vs_oracle(orc, S, mode, order, d, B):
    """B = 1 (one chunk), 2-3 (one proof per chunk), 5 (chunks of 2, 2, 1) of the module pipeline."""
    log_n, k = 8, 11
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code, 0)
    msgs, codes, roots, fin, _, t, out = run_chain(enc, log_n, S, B, d, k, order, mode, 40 + S)
    host_t = np64(t)
    for b in range(B):
        c_ref, r_ref, f_ref, p_ref = orc.commit_prove(code, msgs[b], host_t[b], k, d, order, 40 + S + b, mode)
        assert np.array_equal(np64(codes[b]).reshape(c_ref.shape), c_ref), b
        assert np.array_equal(roots[b].cpu().numpy(), r_ref), b
        assert bytes(fin[b].cpu().numpy()) == f_ref, b
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(p_ref[key].shape), p_ref[key]), (key, b)
    enc.close()


def test_chain_nodes_and_adversarial_tables(orc):
    log_n, S, B, d, k = 9, 4, 2, 2, 14
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code, 0)
    msgs, codes, roots, fin, nd, t, out = run_chain(enc, log_n, S, B, d, k, 0, 0, 7, "adversarial", nodes=True)
    host_t = np64(t)
    for b in range(B):
        c_ref, r_ref, f_ref, p_ref = orc.commit_prove(code, msgs[b], host_t[b], k, d, 0, 7 + b)
        for s in range(S):
            _, nodes_ref = orc.merkle(c_ref[s].astype("<u8").view(np.uint8).reshape(-1, 64), log_n)
            assert np.array_equal(nd[b, s].cpu().numpy(), nodes_ref), (b, s)
        assert bytes(fin[b].cpu().numpy()) == f_ref
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(p_ref[key].shape), p_ref[key]), (key, b)
    enc.close()


def test_chain_argument_errors():
    code = inputs.gen_code(7, 6)
    enc = bzk.Encoder(code, 0)
    t = torch.zeros((1, 1, 16, 4), dtype=torch.int64, device="cuda")
    out = bzk.Prover.alloc_outputs(1, 4, 1)
    sb = bzk.make_batch(4, 1, 0, 0, 1, 0, None, t, 0, 0, out["round_evals"], out["challenges"], out["final_evals"],
                        out["claims"])
    buf = torch.zeros((1, 3, 256, 4), dtype=torch.int64, device="cuda")
    r = torch.zeros((3, 32), dtype=torch.uint8, device="cuda")
    for S in (0, 3):
        c = bzk.bzk_commit(S, 0, buf.data_ptr(), r.data_ptr(), None, r.data_ptr())
        with pytest.raises(bzk.BzkError) as e:
            bzk.bzk_commit_prove(enc.ctx, enc.enc, c, sb)
        assert e.value.status == bzk.BZK_EINVAL
    enc.close()


PIPE_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
sys.path.insert(0, {root!r} + "/tests")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
from test_gpu_chain import run_chain, np64, KEYS
oracle.build()
log_n, S, B, d, k = 8, 2, 5, 2, 11
code = inputs.gen_code(log_n, 6)
enc = bzk.Encoder(code, 0)
msgs, codes, roots, fin, _, t, out = run_chain(enc, log_n, S, B, d, k, 1, 0, 90)
host_t = np64(t)
for b in range(B):
    c_ref, r_ref, f_ref, p_ref = oracle.commit_prove(code, msgs[b], host_t[b], k, d, 1, 90 + b)
    assert np.array_equal(np64(codes[b]).reshape(c_ref.shape), c_ref), b
    assert bytes(fin[b].cpu().numpy()) == f_ref, b
    for key in KEYS:
        assert np.array_equal(np64(out[key][b]).reshape(p_ref[key].shape), p_ref[key]), (key, b)
enc.close()
print("pipeline ok")
"""


@pytest.mark.parametrize("chunks", [2, 4])
def test_chain_module_pipeline(chunks):
    """BZK_CHAIN_CHUNKS > 1: chunks of proofs flow through encode / Merkle / sum-check on three streams
    (B = 5: chunks of 3 + 2 and 2 + 2 + 1); every output bit-exact."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, BZK_CHAIN_CHUNKS=str(chunks))
    r = subprocess.run([sys.executable, "-c", PIPE_SCRIPT.format(root=root)], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0 and "pipeline ok" in r.stdout, r.stdout + r.stderr
