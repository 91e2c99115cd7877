"""Full-field and adversarial inputs (VERDICT r1 "what's weak" #1, #2).

1. Sum-check parity, bit-exact against the oracle, on tables that reach the top of the field:
   `uniform` (now over all of [0, p)), and `adversarial` (per table: [p - 2^16, p), all p - 1,
   alternating 0 / p - 1, the band [2^253, 2^253 + 2^252), or a per-element mix of those, 0 and
   uniform) -- d = 1..4, both orders, k in {1, 5, 9, 10, 13, 16} (tail-only, first tail round 2,
   round 1 + one fused round, several fused rounds, multi-CTA); Goldilocks likewise.
2. The lazy hot-path primitives against Python integers at the operand bounds their comments
   claim (field.cuh, sumcheck.cuh, gl.cuh): both the congruence and the bound of the raw result.
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
GL = bzk.BZK_F_FIELD_GOLDILOCKS
P = int.from_bytes(b"".join(x.to_bytes(8, "little") for x in inputs.P_BN254), "little")
PGL = inputs.P_GL
R = 1 << 256


def np64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def limbs(vals):
    a = np.zeros((len(vals), 4), dtype=np.uint64)
    for i, v in enumerate(vals):
        for j in range(4):
            a[i, j] = (v >> (64 * j)) & (2**64 - 1)
    return a


def ints(a):
    a = a.reshape(-1, 4)
    return [int(a[i, 0]) | int(a[i, 1]) << 64 | int(a[i, 2]) << 128 | int(a[i, 3]) << 192 for i in range(a.shape[0])]


def dev(vals):
    return torch.from_numpy(limbs(vals).view(np.int64)).cuda()


@pytest.fixture(scope="module")
def prover():
    p = bzk.Prover(0)
    yield p
    p.close()


# ---------------------------------------------------------------- generator

@pytest.mark.parametrize("dist", ["uniform", "adversarial", "vml"])
def test_generator_twin_full_range(dist):
    for (B, d, k, I) in [(4, 3, 7, 0), (2, 2, 9, 1000), (3, 4, 0, 7)]:
        t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(t, B, d, k, I, dist)
        assert np.array_equal(np64(t), inputs.gen_tables(B, d, k, I, dist))


@pytest.mark.parametrize("dist", ["gl", "gl_adversarial"])
def test_gl_generator_twin_full_range(dist):
    for (B, d, k, I) in [(4, 3, 7, 0), (2, 2, 9, 1000), (3, 1, 0, 5)]:
        t = torch.empty((B, d, 1 << k), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(t, B, d, k, I, dist)
        assert np.array_equal(np64(t), inputs.gen_tables_gl(B, d, k, I, dist=dist))


# ---------------------------------------------------------------- sum-check parity at the top of the field

SWEEP = [(d, k) for d in (1, 2, 3, 4) for k in (1, 5, 9, 10, 13, 16)]


@pytest.mark.parametrize("dist", ["uniform", "adversarial"])
@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d,k", SWEEP)
def test_sweep_full_field(prover, orc, d, k, order, dist):
    B = 6 if k <= 10 else 3
    I = 7000 + 17 * k + d          # different adversarial table modes per case
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, I, dist)
    out = prover.prove(t, k, d, order, first_index=I, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    for b in range(B):
        ref = orc.prove(host[b], k, d, order, SEED, I + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)


def test_adversarial_modes_cover_the_bounds():
    """The adversarial draw of the sweep really contains every mode (so the sweep sees them)."""
    seen = set()
    for k in (5, 9, 10, 13):
        for d in (1, 2, 3, 4):
            I = 7000 + 17 * k + d
            t = inputs.gen_tables(6 if k <= 10 else 3, d, min(k, 9), I, "adversarial")
            v = ints(t)
            seen |= {"p-1" for x in v if x == P - 1} | {"0" for x in v if x == 0}
            seen |= {"top" for x in v if P - (1 << 16) <= x < P - 1}
            seen |= {"band" for x in v if (1 << 253) <= x < (1 << 253) + (1 << 252)}
            seen |= {"low" for x in v if 0 < x < (1 << 253)}
    assert seen == {"p-1", "0", "top", "band", "low"}


@pytest.mark.parametrize("order", [0, 1])
def test_all_pm1_and_alternating_tables(prover, orc, order):
    """Hand-built extremes: every entry p - 1; alternating 0 / p - 1; the two mixed per table."""
    k, d = 13, 3
    t = torch.zeros((3, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    pm1 = torch.from_numpy(limbs([P - 1]).view(np.int64)[0]).cuda()
    t[0] = pm1
    t[1, :, 1::2] = pm1
    t[2, 0] = pm1
    t[2, 1, 0::2] = pm1
    t[2, 2, 1::2] = pm1
    out = prover.prove(t, k, d, order, first_index=3, flags=bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    for b in range(3):
        ref = orc.prove(host[b], k, d, order, SEED, 3 + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)


@pytest.mark.parametrize("dist", ["gl", "gl_adversarial"])
@pytest.mark.parametrize("order", [0, 1])
@pytest.mark.parametrize("d,k", [(d, k) for d in (1, 2, 3, 4) for k in (1, 5, 9, 10, 13, 16)])
def test_gl_sweep_full_field(prover, orc, d, k, order, dist):
    B = 4 if k <= 10 else 2
    I = 9000 + 17 * k + d
    t = torch.empty((B, d, 1 << k), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, I, dist)
    out = prover.prove(t, k, d, order, first_index=I, flags=GL | bzk.BZK_F_PRESERVE_INPUT)
    torch.cuda.synchronize()
    host = np64(t)
    for b in range(B):
        ref = orc.gl_prove(host[b], k, d, order, SEED, I + b)
        for key in KEYS:
            assert np.array_equal(np64(out[key][b]).reshape(ref[key].shape), ref[key]), (key, b)


# ---------------------------------------------------------------- lazy primitives at their bounds

def run_op(op, a, b):
    A, Bt = dev(a), dev(b)
    n = len(a)
    out = torch.empty((n, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_debug_field(op, n, A, Bt, out)
    torch.cuda.synchronize()
    return ints(np64(out))


def edge_below(bound, rng, n):
    """values in [0, bound): the extremes bound-1, bound-2, multiples of p nearby, and random"""
    e = [bound - 1, bound - 2, 0, 1, P - 1, P, P + 1, 2 * P - 1, 2 * P, 3 * P - 1, 3 * P, 4 * P - 1,
         (1 << 253), (1 << 254) - 1, (1 << 255), R - 1]
    e = [x for x in e if 0 <= x < bound]
    e += [bound - 1 - (int.from_bytes(rng.bytes(4), "little")) for _ in range(16)]
    e += [int.from_bytes(rng.bytes(32), "little") % bound for _ in range(n)]
    return e


def pairs(xs, ys):
    return [x for x in xs for _ in ys], [y for _ in xs for y in ys]


RINV = pow(R, -1, P)


@pytest.mark.parametrize("xb,yb", [(2 * P, 2 * P), (4 * P, P)])
def test_mont_mul_lz_bounds(xb, yb):
    rng = np.random.default_rng(1)
    a, b = pairs(edge_below(xb, rng, 40), edge_below(yb, rng, 40))
    got = run_op(7, a, b)
    for x, y, r in zip(a, b, got):
        assert r % P == x * y * RINV % P
        assert r * R < x * y + P * R and r < 1.76 * P, (x, y, r)     # t = (x y + q p) / R, q < R


@pytest.mark.parametrize("xb,yb", [(2 * P, 2 * P), (P, R)])
def test_mont_mul2_lz_bounds(xb, yb):
    rng = np.random.default_rng(2)
    a, b = pairs(edge_below(xb, rng, 30), edge_below(yb, rng, 30))
    got = run_op(8, a, b)
    n = len(a)
    lim = 2.52 * P if xb == 2 * P else 3 * P
    for i in range(n):
        s = a[i] * b[i] + a[n - 1 - i] * b[n - 1 - i]
        assert got[i] % P == s * RINV % P
        assert got[i] < lim and got[i] < R, i


def test_fixmul_lz_bounds():
    """fixmul_lz: x any 256-bit value, r canonical -> r x (mod p), result < p (1 + 2^-29)."""
    rng = np.random.default_rng(3)
    xs = edge_below(R, rng, 60)
    rs = [0, 1, 2, P - 1, P - 2, (1 << 253), P // 2] + [int.from_bytes(rng.bytes(32), "little") % P for _ in range(20)]
    a, b = pairs(xs, rs)
    got = run_op(9, a, b)
    for x, r, g in zip(a, b, got):
        assert g % P == x * r % P
        assert g < P + (P >> 29), (x, r, g)


def test_fold_fx_bounds():
    """The hot-loop fold a + r (b - a) on lazy inputs a, b < 2p: congruent and < 2p."""
    rng = np.random.default_rng(4)
    xs = edge_below(2 * P, rng, 20)
    a, b = pairs(xs, xs)
    rs = [[0, 1, P - 1, (1 << 253)][i % 4] if i < 64 else int.from_bytes(rng.bytes(32), "little") % P
          for i in range(len(a))]
    got = run_op(16, a, b + rs)
    for x, y, r, g in zip(a, b, rs, got):
        assert g % P == (x + r * (y - x)) % P
        assert g < 2 * P, (x, y, r, g)


def test_mul_acc_and_acc17_to_fe():
    """544-bit unreduced sums of 64 products of operands up to 2^256 - 1 (beyond the 4p the loop
    guarantees) reduce to the canonical S R^-1; raw 544-bit accumulators up to 2^544 - 1 too."""
    rng = np.random.default_rng(5)
    n = 512
    a = [R - 1 - (i % 3) for i in range(64)] + edge_below(R, rng, n - 64 - 16)
    b = [R - 1] * 64 + edge_below(4 * P, rng, n - 64 - 16)
    a, b = a[:n], b[:n]
    got = run_op(10, a, b)
    for i in range(n):
        s = sum(a[(i + j) % n] * b[(i + j) % n] for j in range(64))
        assert got[i] == s * RINV % P, i
    raw_lo = [R - 1, 0, R - 1, P, 1 << 255] + edge_below(R, rng, 40)
    raw_hi = [R - 1, R - 1, 0, P - 1, 1 << 200] + edge_below(R, rng, 40)
    got = run_op(11, raw_lo, raw_hi)
    for lo, hi, g in zip(raw_lo, raw_hi, got):
        v = lo + (hi << 256) + ((lo >> 224) << 512)
        assert g == v * RINV % P


def test_lz_sub_red_add_exact():
    rng = np.random.default_rng(6)
    xs = edge_below(2 * P, rng, 30)
    a, b = pairs(xs, xs)
    for g, x, y in zip(run_op(12, a, b), a, b):      # lz_sub(b, a) = b + 2p - a, exact, in (0, 4p)
        assert g == y + 2 * P - x and 0 < g < 4 * P
    ys = edge_below(4 * P, rng, 200)
    for g, x in zip(run_op(13, ys, ys), ys):         # lz_red: exact, < 2p
        assert g == (x - 2 * P if x >= 2 * P else x)
    for g, x, y in zip(run_op(15, a, b), a, b):      # lz_add exact (< 4p < 2^256)
        assert g == x + y


def test_acc9_to_fe():
    rng = np.random.default_rng(7)
    lo = edge_below(R, rng, 60)
    hi = [R - 1, 0xFFFFFFFF, 1, 0] + [int(x) for x in rng.integers(0, 2**32, size=len(lo) - 4)]
    for g, x, h in zip(run_op(14, lo, hi), lo, hi):
        assert g == (x + ((h & 0xFFFFFFFF) << 256)) % P


# ---------------------------------------------------------------- Goldilocks primitives

def gl_run(op, a, b):
    A = torch.from_numpy(np.array(a, dtype=np.uint64).view(np.int64)).cuda()
    Bt = torch.from_numpy(np.array(b, dtype=np.uint64).view(np.int64)).cuda()
    out = torch.empty(len(a), dtype=torch.int64, device="cuda")
    bzk.bzk_debug_gl(op, len(a), A, Bt, out)
    torch.cuda.synchronize()
    return [int(x) for x in np64(out)]


def gl_edges(rng, bound, n):
    e = [0, 1, 2, PGL - 1, PGL - 2, 2**63, 2**63 - 1, 2**32, 2**32 - 1, 2**64 - 2**32, PGL]
    e = [x for x in e if x < bound]
    return e + [int(x) % bound for x in rng.integers(0, 2**63, size=n, dtype=np.int64)] + \
        [(bound - 1 - int(x)) for x in rng.integers(0, 2**16, size=8)]


def test_gl_canonical_ops():
    rng = np.random.default_rng(8)
    xs = gl_edges(rng, PGL, 40)
    a, b = pairs(xs, xs)
    assert gl_run(0, a, b) == [(x + y) % PGL for x, y in zip(a, b)]
    assert gl_run(1, a, b) == [(x - y) % PGL for x, y in zip(a, b)]
    assert gl_run(2, a, b) == [(x * y) % PGL for x, y in zip(a, b)]
    rs = [int(x) % PGL for x in rng.integers(0, 2**63, size=len(a), dtype=np.int64)]
    rs[:4] = [0, 1, PGL - 1, 2**63]
    assert gl_run(5, a, b + rs) == [(x + r * (y - x)) % PGL for x, y, r in zip(a, b, rs)]


def test_gl_lazy_ops():
    rng = np.random.default_rng(9)
    xs = gl_edges(rng, 2**64, 40)
    a, b = pairs(xs, xs)
    # add_lazy: x < 2^64 (a lazy sum), y canonical -- how eval_pair uses it (v + delta)
    ya = gl_edges(rng, PGL, 40)
    xa, yb = pairs(xs, ya)
    for g, x, y in zip(gl_run(3, xa, yb), xa, yb):
        assert g % PGL == (x + y) % PGL and g < 2**64
    assert gl_run(4, a, b) == [((x << 64) + y) % PGL for x, y in zip(a, b)]   # reduce128(hi, lo)
    n = 256
    u = ([2**64 - 1] * 64 + gl_edges(rng, 2**64, n))[:n]
    v = ([2**64 - 1] * 64 + gl_edges(rng, 2**64, n))[:n]
    assert gl_run(6, u, v) == [sum(u[(i + j) % n] * v[(i + j) % n] for j in range(64)) % PGL for i in range(n)]
    tops = [2**32 - 1, 0, 1] + [int(x) for x in rng.integers(0, 2**32, size=len(a) - 3)]
    got = gl_run(7, a, b + tops)
    assert got == [(x + (y << 64) + ((t & 0xFFFFFFFF) << 128)) % PGL for x, y, t in zip(a, b, tops)]
