"""CPU tests of the seeded input generator (inputs.py): canonical over the WHOLE
field, the adversarial modes present, independence of batch composition.  The device twin
(gen.cuh) is compared word for word in tests/test_gpu_fullrange.py."""
import numpy as np

from paper_conf_asplos_lucw0cz25_b200 import inputs

P = int.from_bytes(b"".join(x.to_bytes(8, "little") for x in inputs.P_BN254), "little")


def ints(t):
    t = t.reshape(-1, 4)
    return [int(r[0]) | int(r[1]) << 64 | int(r[2]) << 128 | int(r[3]) << 192 for r in t]


def test_bound_constants_are_the_moduli():
    # BN254 r(u) = 36u^4 + 36u^3 + 18u^2 + 6u + 1, u = 4965661367192848881 (tests/golden/bn254_fr.txt)
    u = 4965661367192848881
    assert P == 36 * u**4 + 36 * u**3 + 18 * u**2 + 6 * u + 1
    assert inputs.P_GL == 2**64 - 2**32 + 1


def test_uniform_is_canonical_and_reaches_the_top():
    v = ints(inputs.gen_tables(8, 3, 9, 0, "uniform"))
    assert max(v) < P
    top = sum(x >= (1 << 253) for x in v) / len(v)
    assert 0.22 < top < 0.29            # (p - 2^253) / 2^254 = 0.256 of the 254-bit draws
    assert max(v) > P - P // 1000       # values close to p occur


def test_canonical_subtraction_matches_integers():
    # the raw 254-bit draw minus p where >= p, checked against Python integers
    words = np.array([[2**64 - 1] * 3 + [2**64 - 1], list(inputs.P_BN254), [0, 0, 0, 0],
                      [inputs.P_BN254[0] - 1] + list(inputs.P_BN254[1:])], dtype=np.uint64)
    out = inputs._canonical_254(words)
    for w, o in zip(ints(words), ints(out)):
        w &= (1 << 254) - 1
        assert o == (w - P if w >= P else w)


def test_adversarial_modes():
    seen = {"p-1": 0, "0": 0, "top": 0, "band": 0, "alternating": 0, "uniform-low": 0}
    for I in range(0, 60):
        t = inputs.gen_tables(1, 2, 6, I, "adversarial")[0]
        for m in range(2):
            v = ints(t[m])
            assert max(v) < P
            if all(x == P - 1 for x in v):
                seen["p-1"] += 1
            if all(x == (0 if j % 2 == 0 else P - 1) for j, x in enumerate(v)):
                seen["alternating"] += 1
            seen["top"] += sum(P - (1 << 16) <= x < P - 1 for x in v)
            seen["band"] += sum((1 << 253) <= x < (1 << 253) + (1 << 252) for x in v)
            seen["0"] += sum(x == 0 for x in v)
            seen["uniform-low"] += sum(0 < x < (1 << 253) for x in v)
    assert all(c > 0 for c in seen.values()), seen


def test_gl_full_range_and_adversarial():
    g = inputs.gen_tables_gl(6, 2, 10, 0)
    assert g.max() < inputs.P_GL and (g >= 2**63).mean() > 0.45
    a = inputs.gen_tables_gl(40, 2, 5, 0, dist="gl_adversarial")
    assert a.max() < inputs.P_GL
    assert (a == inputs.P_GL - 1).any() and (a == 0).any() and (a >= 2**63).any()


def test_batch_composition_independence():
    full = inputs.gen_tables(5, 2, 6, 10, "adversarial")
    assert np.array_equal(full[2:4], inputs.gen_tables(2, 2, 6, 12, "adversarial"))
    assert np.array_equal(full[[1, 4]], inputs.gen_tables(2, 2, 6, dist="adversarial", indices=[11, 14]))
