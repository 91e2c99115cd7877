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


def test_m0_and_g2_full_size(orc):
    """m0 (paper shape: 1024 x d=1, k=20, MSB) and g2 (Goldilocks 1024 x d=2, k=20) at full size in
    bench.py's launch configuration: sampled proofs vs the oracle."""
    rng = np.random.default_rng(4)
    sample = sorted({0, 1023, *rng.choice(1024, size=2, replace=False).tolist()})
    torch.cuda.empty_cache()
    # m0
    t = torch.empty((1024, 1, 1 << 20, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, 1024, 1, 20, 0, "uniform")
    p = bzk.Prover(0)
    out = p.prove(t, 20, 1, 1, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.sync()
    del t
    for i in sample:
        ref = orc.prove(inputs.gen_tables(1, 1, 20, first_index=i)[0], 20, 1, 1, SEED, i)
        for key in KEYS:
            assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), ("m0", key, i)
    torch.cuda.empty_cache()
    # g2
    t = torch.empty((1024, 2, 1 << 20), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, 1024, 2, 20, 0, "gl")
    out = p.prove(t, 20, 2, 0, flags=bzk.BZK_F_PRESERVE_INPUT | bzk.BZK_F_FIELD_GOLDILOCKS)
    p.sync()
    host = np64(t[sample])
    for n, i in enumerate(sample):
        ref = orc.gl_prove(host[n], 20, 2, 0, SEED, i)
        for key in KEYS:
            assert np.array_equal(np64(out[key][i]).reshape(ref[key].shape), ref[key]), ("g2", key, i)
    p.close()
    del t
    torch.cuda.empty_cache()


def test_vml_image_shapes(orc):
    """configs[3]: the 32 sum-checks of one VGG-16/CIFAR-10-shaped image (k per layer as bench.py),
    streamed from pinned host memory through bzk_prove_ragged, every proof vs the oracle."""
    ks = [16, 16, 15, 15, 14, 14, 14, 13, 13, 13, 11, 11, 11, 9, 9, 9]
    p = bzk.Prover(0)
    jobs, outs, tabs = [], [], []
    for li, k in enumerate(ks):
        I = 5000 + 2 * li
        t = torch.empty((2, 2, 1 << k, 4), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(t, 2, 2, k, I, "vml")
        ht = t.cpu().pin_memory()
        o = bzk.Prover.alloc_outputs(2, k, 2, device="cpu", pin=True)
        tabs.append(ht)
        outs.append(o)
        jobs.append(p.batch(ht, k, 2, 0, None, I, 0, o))
    bzk.bzk_prove_ragged(p.ctx, jobs)
    for li, k in enumerate(ks):
        host = tabs[li].numpy().view(np.uint64)
        for b in range(2):
            ref = orc.prove(host[b], k, 2, 0, SEED, 5000 + 2 * li + b)
            for key in KEYS:
                assert np.array_equal(outs[li][key][b].numpy().view(np.uint64).reshape(ref[key].shape), ref[key])
    p.close()


def test_mk20_full_size(orc):
    """NEXT-3 at bench.py's mk20 call: 256 trees x 2^20 blocks, node arrays on the device (one
    bzk_merkle call over the whole batch).  Sampled trees recomputed by the oracle (every node);
    every root checked against the sampled-leaf authentication paths is implied by the node check."""
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    B, n = 256, 20
    blocks = torch.empty((B, 1 << n, 64), dtype=torch.uint8, device="cuda")
    bzk.bzk_generate_blocks(blocks, B, n, 0)
    mb = bzk.MerkleBuilder(0)
    roots, nodes = mb.build(blocks, n, bzk.BZK_MERKLE_COMPRESS)
    torch.cuda.synchronize()
    for b in (0, 137, 255):
        exp_root, exp_nodes = orc.merkle(inputs.gen_blocks(1, n, first_index=b)[0], n, 0)
        assert bytes(roots[b].cpu().numpy()) == exp_root
        assert np.array_equal(nodes[b].cpu().numpy(), exp_nodes)
    mb.close()


def test_enc20_full_size(orc):
    """NEXT-4 at bench.py's enc20 call: 256 codewords of 2^20 elements in one bzk_encode; sampled
    codewords recomputed by the oracle element by element."""
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    B, log_n = 256, 20
    n = 1 << log_n
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code, 0)
    msgs = torch.empty((B, 1, n, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(msgs, B, 1, log_n, 0, "uniform")
    codes = torch.empty((B, 2 * n, 4), dtype=torch.int64, device="cuda")
    codes[:, :n].copy_(msgs[:, 0])
    enc.encode(codes)
    torch.cuda.synchronize()
    for b in (0, 255):
        m = inputs.gen_tables(1, 1, log_n, first_index=b)[0, 0]
        assert np.array_equal(codes[b].cpu().numpy().view(np.uint64), orc.encode(code, m))
    enc.close()
