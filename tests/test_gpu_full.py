"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

configs[1]: 1024 proofs, d = 2, k = 20 (device-resident, PRESERVE mode -- exactly bench.py's call).
configs[2]: 256 proofs, d = 3, k = 22 (consume mode: 96 GiB input + 48 GiB scratch).
Sampled proofs (first, last, random) are recomputed by the oracle and compared bit-exactly; every
proof of the batch is checked by the reference verifier (round invariant, transcript, final check).
"""
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


def run_full(orc, B, d, k, order, flags, sample):
    torch.cuda.empty_cache()
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 0, "uniform")
    p = bzk.Prover(0)
    out = p.prove(t, k, d, order, flags=flags)
    p.sync()
    del t
    p.close()
    torch.cuda.empty_cache()
    host = {key: np64(out[key]) for key in KEYS}
    # oracle on the sampled proofs (one thread each)
    tabs = np.stack([inputs.gen_tables(1, d, k, first_index=int(i))[0] for i in sample])
    for n, i in enumerate(sample):
        ref = orc.prove(tabs[n], k, d, order, SEED, int(i))
        for key in KEYS:
            assert np.array_equal(host[key][i].reshape(ref[key].shape), ref[key]), (key, i)
    for b in range(B):
        assert orc.verify(k, d, order, SEED, b, host["round_evals"][b], host["challenges"][b],
                          host["final_evals"][b], host["claims"][b]) == 0, b
    return host


def test_config2_full_size(orc):
    rng = np.random.default_rng(2)
    sample = sorted({0, 1023, *rng.choice(1024, size=4, replace=False).tolist()})
    run_full(orc, 1024, 2, 20, 0, bzk.BZK_F_PRESERVE_INPUT, sample)


def test_config3_full_size(orc):
    free, _ = torch.cuda.mem_get_info()
    if free < 150 * 2**30:
        pytest.skip("needs ~150 GiB free device memory")
    rng = np.random.default_rng(3)
    sample = sorted({0, 255, *rng.choice(256, size=2, replace=False).tolist()})
    run_full(orc, 256, 3, 22, 0, 0, sample)
