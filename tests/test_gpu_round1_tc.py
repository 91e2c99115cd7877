"""k_round1_tc (csrc/round1_tc.cuh): round 1 of d = 2 BN254 proofs on the tensor cores -- the sums
g(0), g(1) and the leading coefficient as u8 products over the pairs -- bit-exact against the oracle
(every output of the whole proof, since r_1 and everything after it depends on round 1).

k >= 15 keeps the batches out of k_small (whose single-launch path has its own round 1); the profile
confirms the tensor-core kernel ran.  Cases: both orders, one and several CTAs per proof (last-CTA
ticket), ragged tile counts per CTA, the byte extremes (p - 1 everywhere, alternating 0 / p - 1, the
adversarial generator), and BZK_R1_TC=0 (the CUDA-core k_round) on the same inputs.
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


def prove(p, t, k, order, first_index):
    B = t.shape[0]
    out = bzk.Prover.alloc_outputs(B, k, 2)
    b = p.batch(t, k, 2, order, None, first_index, bzk.BZK_F_PRESERVE_INPUT, out)
    bzk.bzk_prove(p.ctx, b)
    torch.cuda.synchronize()
    return out


def check(orc, host, out, k, order, first_index):
    for b in range(host.shape[0]):
        ref = orc.prove(np.ascontiguousarray(host[b]), k, 2, order, SEED, first_index + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, k, order)


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("k,B,dist", [(15, 1, "uniform"), (16, 3, "adversarial"), (17, 2, "uniform")])
def test_round1_tc_vs_oracle(orc, order, k, B, dist):
    I = 40 + k
    t = torch.empty((B, 2, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 2, k, I, dist)
    p = bzk.Prover(0)
    bzk.bzk_profile_enable(p.ctx, 1)
    out = prove(p, t, k, order, I)
    prof = bzk.bzk_profile_read(p.ctx, 1)
    p.close()
    assert prof["round1_eval"][1] > 0
    check(orc, np64(t), out, k, order, I)


@pytest.mark.parametrize("order", [0, 1])
def test_round1_tc_byte_extremes(orc, order):
    """every entry p - 1 (the largest byte products and anti-diagonal sums), alternating 0 / p - 1,
    and one table zero"""
    k = 15
    N = 1 << k
    pm1 = np.array(inputs.P_BN254, dtype=np.uint64).copy()
    pm1[0] -= 1
    host = np.zeros((3, 2, N, 4), dtype=np.uint64)
    host[0, :, :] = pm1
    host[1, 0, 0::2] = pm1
    host[1, 1, 1::2] = pm1
    host[2, 0, :] = pm1
    t = torch.from_numpy(host.view(np.int64)).cuda()
    p = bzk.Prover(0)
    out = prove(p, t, k, order, 9)
    p.close()
    check(orc, host, out, k, order, 9)


SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r}); sys.path.insert(0, {root!r} + "/tests")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk
from test_gpu_round1_tc import prove, check, np64
oracle.build()
for k, B, order in [(16, 2, 0), (16, 1, 1), (18, 1, 0)]:
    t = torch.empty((B, 2, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 2, k, 70 + k, "adversarial")
    p = bzk.Prover(0)
    out = prove(p, t, k, order, 70 + k)
    p.close()
    check(oracle, np64(t), out, k, order, 70 + k)
print("r1tc ok")
"""


@pytest.mark.parametrize("env", [{"BZK_R1TC_CTAS": "1"}, {"BZK_R1TC_CTAS": "7"}, {"BZK_R1TC_CTAS": "100000"},
                                 {"BZK_R1_TC": "0"}, {"BZK_FTC_SMALL_LOG": "0"}, {"BZK_FTC_SMALL_LOG": "17"},
                                 {"BZK_R1_SW64": "0"}, {"BZK_R1_SW64": "0", "BZK_R1TC_CTAS": "7"},
                                 {"BZK_FUSED_TC": "0", "BZK_R1_TC": "0"}, {"BZK_FUSED_TC": "0", "BZK_TMA": "0"},
                                 {"BZK_FUSED_TC": "0", "BZK_R1_TC": "0", "BZK_TMA": "1"}])
def test_round1_tc_launch_shapes(env):
    """one CTA per proof, 7 CTAs (ragged: 256 tiles -> 37 / 36 per CTA), one CTA per tile, and the
    CUDA-core round 1 (BZK_R1_TC=0); the 2-warp k_fused_tc of the late d = 2 rounds off, and on for
    every fused round (several CTAs per proof); LSB round 1 from separate a / b boxes of 32-byte rows
    instead of one box of 64-byte (a | b) rows; the CUDA-core k_round for round 1 and the fused rounds
    (BZK_FUSED_TC=0, BZK_R1_TC=0) with its TMA staging at the default, off and forced on"""
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT)], env=dict(os.environ, **env),
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "r1tc ok" in r.stdout, r.stdout + r.stderr
