"""The 64-thread CTAs of the late CUDA-core global rounds (api.cu small_round, BZK_SMALL_ROUND_LOG): d = 1
BN254 proofs (k_round without TMA staging) and Goldilocks proofs (k_gl_round), bit-exact against the
oracle with the variant at its default (h <= 2^12), off, and forced on for every fused round (several
CTAs per proof up to 2^15 pairs).  k >= 15 keeps the BN254 batches out of k_small.
"""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
oracle.build()
SEED = inputs.DEFAULT_SEED
KEYS = ("round_evals", "challenges", "final_evals", "claims")
np64 = lambda t: t.detach().cpu().numpy().view(np.uint64)
p = bzk.Prover(0)
for (B, k, order) in [(3, 16, 1), (2, 15, 0)]:          # BN254, d = 1
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 50 + k, "adversarial")
    out = p.prove(t, k, 1, order, first_index=50 + k, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    for b in range(B):
        ref = oracle.prove(np.ascontiguousarray(host[b]), k, 1, order, SEED, 50 + k + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, k, order)
for (B, d, k, order) in [(3, 2, 16, 0), (2, 1, 15, 1), (2, 3, 14, 0)]:   # Goldilocks
    t = torch.empty((B, d, 1 << k), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 7, "gl")
    out = p.prove(t, k, d, order, first_index=7, flags=bzk.BZK_F_FIELD_GOLDILOCKS | bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    for b in range(B):
        ref = oracle.gl_prove(host[b], k, d, order, SEED, 7 + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, k, d, order)
p.close()
print("small rounds ok")
"""


@pytest.mark.parametrize("env", [{}, {"BZK_SMALL_ROUND_LOG": "0"}, {"BZK_SMALL_ROUND_LOG": "15"}])
def test_small_rounds(env):
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT)], env=dict(os.environ, **env),
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and "small rounds ok" in r.stdout, r.stdout + r.stderr
