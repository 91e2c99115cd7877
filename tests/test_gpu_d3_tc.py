"""k_fused_tc<3, ORDER, FIRST> (csrc/fused_tc.cuh): round 1 and the fused rounds of d = 3 BN254 proofs
with the last product of every summed point (eval_one's unreduced 256 x 256-bit product) summed over
the pairs on the tensor cores -- bit-exact against the oracle (every output of the whole proof).

k >= 15 keeps the batches out of k_small.  Cases: both orders, the adversarial and uniform generators,
the byte extremes (p - 1 everywhere, alternating 0 / p - 1, one table zero), several CTA counts per
proof (BZK_PPT_MAX / BZK_CTA_WAVES change the grid; ragged tile counts per warp), and BZK_D3_TC=0 (the
CUDA-core k_round) on the same inputs.
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
D = 3


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def prove(p, t, k, order, first_index, d=D):
    B = t.shape[0]
    out = bzk.Prover.alloc_outputs(B, k, d)
    b = p.batch(t, k, d, order, None, first_index, bzk.BZK_F_PRESERVE_INPUT, out)
    bzk.bzk_prove(p.ctx, b)
    torch.cuda.synchronize()
    return out


def check(orc, host, out, k, order, first_index, d=D):
    for b in range(host.shape[0]):
        ref = orc.prove(np.ascontiguousarray(host[b]), k, d, order, SEED, first_index + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b, k, order)


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("k,B,dist", [(15, 1, "uniform"), (16, 3, "adversarial"), (17, 2, "uniform")])
def test_d3_tc_vs_oracle(orc, order, k, B, dist):
    I = 300 + k
    t = torch.empty((B, D, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, D, k, I, dist)
    p = bzk.Prover(0)
    out = prove(p, t, k, order, I)
    p.close()
    check(orc, np64(t), out, k, order, I)


@pytest.mark.parametrize("order", [0, 1])
def test_d3_tc_byte_extremes(orc, order):
    """every entry p - 1 (the largest byte products), alternating 0 / p - 1 per table, one table zero"""
    k = 15
    N = 1 << k
    pm1 = np.array(inputs.P_BN254, dtype=np.uint64).copy()
    pm1[0] -= 1
    host = np.zeros((3, D, N, 4), dtype=np.uint64)
    host[0, :, :] = pm1
    host[1, 0, 0::2] = pm1
    host[1, 1, 1::2] = pm1
    host[1, 2, 0::2] = pm1
    host[2, 0, :] = pm1
    host[2, 2, :] = pm1
    t = torch.from_numpy(host.view(np.int64)).cuda()
    p = bzk.Prover(0)
    out = prove(p, t, k, order, 11)
    p.close()
    check(orc, host, out, k, order, 11)


SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r}); sys.path.insert(0, {root!r} + "/tests")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk
from test_gpu_d3_tc import prove, check, np64
oracle.build()
for k, B, order in [(16, 2, 0), (16, 1, 1), (18, 1, 0), (17, 3, 1)]:
    t = torch.empty((B, 3, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 3, k, 90 + k, "adversarial")
    p = bzk.Prover(0)
    out = prove(p, t, k, order, 90 + k)
    p.close()
    check(oracle, np64(t), out, k, order, 90 + k)
print("d3tc ok")
"""


@pytest.mark.parametrize("env", [{"BZK_PPT_MAX": "1"}, {"BZK_PPT_MAX": "3", "BZK_CTA_WAVES": "1"},
                                 {"BZK_CTA_WAVES": "16"}, {"BZK_D3_TC": "0"}])
def test_d3_tc_launch_shapes(env):
    """different CTA counts per proof (one pair per thread; 3 pairs per thread -> ragged warp tile
    counts; many CTAs), and the CUDA-core rounds (BZK_D3_TC=0)"""
    r = subprocess.run([sys.executable, "-c", SCRIPT.format(root=ROOT)], env=dict(os.environ, **env),
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "d3tc ok" in r.stdout, r.stdout + r.stderr
