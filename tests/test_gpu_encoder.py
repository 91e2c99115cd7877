"""GPU parity of the batched linear-time encoder against the CPU oracle.

Every codeword element is compared bit-exactly with oracle.encode on the same graphs and messages:
base-only codes (levels = 0), one and several recursion levels, odd batch sizes (the kernel pairs
codewords), small-int / zero / boundary (p - 1) messages, device and pinned-host buffers (loader waves),
and at the bench size (n = 2^20) on sampled codewords.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402

P = 0x30644E72E131A029B85045B68181585D2833E84879B9709143E1F593F0000001


def msgs_np(B, log_n, first=0):
    return inputs.gen_tables(B, 1, log_n, first_index=first)[:, 0]          # [B][n][4] u64


def codes_dev(m):
    B, n, _ = m.shape
    c = torch.zeros((B, 2 * n, 4), dtype=torch.int64, device="cuda")
    c[:, :n] = torch.from_numpy(m.view(np.int64)).cuda()
    return c


def check(orc, code, m, got):
    exp = orc.encode_batch(code, m)
    g = got.cpu().numpy().view(np.uint64)
    bad = np.argwhere(np.any(g != exp, axis=-1))
    assert bad.size == 0, f"codeword mismatches at (b, i) {bad[:8].tolist()} of {bad.shape[0]}"


@pytest.mark.parametrize("log_n,B", [(6, 3), (7, 2), (8, 5), (10, 4), (12, 3), (13, 1)])
def test_encoder_sweep(orc, log_n, B):
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code)
    m = msgs_np(B, log_n, first=log_n)
    c = codes_dev(m)
    enc.encode(c)
    torch.cuda.synchronize()
    check(orc, code, m, c)
    enc.close()


def test_encoder_special_messages(orc):
    log_n = 9
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code)
    n = 1 << log_n
    m = np.zeros((4, n, 4), np.uint64)
    m[1] = orc.to_limbs([P - 1] * n)                                       # boundary values
    m[2] = inputs.gen_tables(1, 1, log_n, dist="smallint")[0, 0]            # 8-bit values
    m[3, 17] = orc.to_limbs([1])[0]                                         # a unit vector
    c = codes_dev(m)
    enc.encode(c)
    torch.cuda.synchronize()
    check(orc, code, m, c)
    assert not c[0].any()                                                   # Enc(0) = 0
    enc.close()


def test_encoder_host_memory_waves(orc):
    log_n, B = 11, 9
    code = inputs.gen_code(log_n, 6)
    n = 1 << log_n
    enc = bzk.Encoder(code, workspace_limit=2 * 2 * (2 * n * 32) * 2 + (1 << 20))
    m = msgs_np(B, log_n, first=50)
    host = torch.zeros((B, 2 * n, 4), dtype=torch.int64).pin_memory()
    host[:, :n] = torch.from_numpy(m.view(np.int64))
    host[:, n:] = 7                                                          # garbage the encoder overwrites
    enc.encode(host)
    check(orc, code, m, host)
    enc.close()


def test_encoder_bench_size_sampled(orc):
    """n = 2^20 (the bench's code, 7 levels), 4 codewords; two of them recomputed by the oracle."""
    log_n, B = 20, 4
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code)
    m = msgs_np(B, log_n, first=900)
    c = codes_dev(m)
    enc.encode(c)
    torch.cuda.synchronize()
    for b in (0, 3):
        exp = orc.encode(code, m[b])
        assert np.array_equal(c[b].cpu().numpy().view(np.uint64), exp)
    enc.close()


def test_encoder_argument_errors():
    code = inputs.gen_code(8, 6)
    ctx = bzk.bzk_create(0)
    bad = dict(code)
    bad["A"] = [dict(code["A"][0], rows=code["A"][0]["rows"] + 1)]
    with pytest.raises(bzk.BzkError):
        bzk.bzk_encoder_create(ctx, bad)
    bad = dict(code)
    a0 = dict(code["A"][0])
    col = a0["col"].copy()
    col[3] = a0["cols"]                                                       # column out of range
    a0["col"] = col
    bad["A"] = [a0]
    with pytest.raises(bzk.BzkError):
        bzk.bzk_encoder_create(ctx, bad)
    enc = bzk.bzk_encoder_create(ctx, code)
    c = torch.zeros((1, 512, 4), dtype=torch.int64, device="cuda")
    with pytest.raises(bzk.BzkError):
        bzk.bzk_encode(ctx, enc, c, 0)
    bzk.bzk_encoder_destroy(enc)
    bzk.bzk_destroy(ctx)
