"""GPU parity for the Goldilocks field instance (BZK_F_FIELD_GOLDILOCKS):
CUDA path vs the oracle's Goldilocks prover, every output bit-exact."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

SEED = inputs.DEFAULT_SEED
KEYS = ("round_evals", "challenges", "final_evals", "claims")
GL = bzk.BZK_F_FIELD_GOLDILOCKS


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def gl_tables(B, d, k, I=0):
    t = torch.empty((B, d, 1 << k), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, I, "gl")
    return t


@pytest.fixture(scope="module")
def prover():
    p = bzk.Prover(0)
    yield p
    p.close()


def check(orc, host, out, k, d, order, I, given=None):
    for b in range(host.shape[0]):
        ref = orc.gl_prove(host[b], k, d, order, SEED, I + b, given=None if given is None else given[b])
        for key in KEYS:
            got = np64(out[key][b]).reshape(ref[key].shape)
            assert np.array_equal(got, ref[key]), (key, b, k, d, order)


def test_gl_generator_matches_host_twin():
    for (B, d, k, I) in [(2, 2, 6, 0), (1, 3, 9, 77), (3, 1, 0, 5)]:
        assert np.array_equal(np64(gl_tables(B, d, k, I)), inputs.gen_tables_gl(B, d, k, I))


@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d,k", [(d, k) for d in (1, 2, 3, 4) for k in (0, 1, 3, 8, 9, 10, 12, 13)])
def test_gl_sweep(prover, orc, d, k, order):
    B, I = 3, 40 + k
    t = gl_tables(B, d, k, I)
    out = prover.prove(t, k, d, order, first_index=I, flags=GL)
    torch.cuda.synchronize()
    check(orc, inputs.gen_tables_gl(B, d, k, I), out, k, d, order, I)


@pytest.mark.parametrize("k", [15, 17])
def test_gl_many_ctas(prover, orc, k):
    B, d = 4, 2
    t = gl_tables(B, d, k, 9)
    out = prover.prove(t, k, d, 0, first_index=9, flags=GL | bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    check(orc, np64(t), out, k, d, 0, 9)


def test_gl_given_challenges(prover, orc):
    B, d, k = 2, 2, 11
    t = gl_tables(B, d, k, 3)
    rng = np.random.default_rng(1)
    r = rng.integers(0, 2**63, size=(B, k), dtype=np.uint64)
    out = bzk.Prover.alloc_outputs_gl(B, k, d)
    out["challenges"].copy_(torch.from_numpy(r.view(np.int64)))
    b = prover.batch(t, k, d, 1, None, 3, GL | bzk.BZK_F_GIVEN_CHALLENGES | bzk.BZK_F_PRESERVE_INPUT, out)
    bzk.bzk_prove(prover.ctx, b)
    torch.cuda.synchronize()
    check(orc, np64(t), out, k, d, 1, 3, given=r)


def test_gl_host_tables_validate_and_waves(orc):
    B, d, k = 5, 2, 14
    t = gl_tables(B, d, k)
    p = bzk.Prover(0, workspace_limit=6 * (1 << k) * 8 * 2)
    out_h = bzk.Prover.alloc_outputs_gl(B, k, d, device="cpu", pin=True)
    p.prove(t.cpu().pin_memory(), k, d, 0, out=out_h, flags=GL | bzk.BZK_F_VALIDATE)
    torch.cuda.synchronize()
    check(orc, np64(t), out_h, k, d, 0, 0)
    t[1, 0, 5] = -1                      # 2^64 - 1 >= p
    with pytest.raises(bzk.BzkError) as e:
        p.prove(t, k, d, 0, flags=GL | bzk.BZK_F_VALIDATE)
    assert e.value.status == bzk.BZK_ENONCANON
    p.close()
