"""Pins of the oracle's section-4 chain (oracle.commit_prove, R25) against
independent Python: the final root by the recursive definition over the codeword roots (oracle/py
merkle, SHA-256 constants derived from first principles), each codeword root likewise, and the
sum-check transcript seeded with that root by the Python cross-oracle (oracle/py/sumcheck.py)."""
import numpy as np
import pytest

from paper_conf_asplos_lucw0cz25_b200 import inputs


@pytest.mark.parametrize("S,mode", [(1, 0), (2, 0), (4, 1), (8, 0)])
def test_chain_matches_independent_composition(orc, S, mode):
    from oracle.py import merkle as pm
    from oracle.py import sumcheck as ps
    log_n, k, d, I = 7, 5, 2, 11
    code = inputs.gen_code(log_n, 6)
    segs = inputs.gen_tables(S, 1, log_n, first_index=100)[:, 0]
    tabs = inputs.gen_tables(1, d, k, first_index=I, dist="adversarial")[0]
    codes, roots, final, proof = orc.commit_prove(code, segs, tabs, k, d, 0, I, mode)
    assert np.array_equal(codes, orc.encode_batch(code, segs))
    for s in range(S):
        blocks = [codes[s].astype("<u8").tobytes()[64 * x:64 * (x + 1)] for x in range(1 << log_n)]
        assert roots[s].tobytes() == pm.merkle_root_recursive(blocks, mode)
    # the roots are the LEAVES of the top tree: level 1 = H(root_2j || root_2j+1)
    level = [roots[s].tobytes() for s in range(S)]
    while len(level) > 1:
        level = [pm.H(level[2 * j] + level[2 * j + 1], mode) for j in range(len(level) // 2)]
    assert final == level[0]
    T = [orc.from_limbs(tabs[m]) for m in range(d)]
    evals, chals, finals, H = ps.prove(T, k, final, I, 0)
    assert orc.from_limbs(proof["challenges"]) == chals
    assert orc.from_limbs(proof["round_evals"].reshape(-1, 4)) == [v for g in evals for v in g]
    assert orc.from_limbs(proof["final_evals"]) == finals and orc.from_limbs(proof["claims"].reshape(1, 4)) == [H]


def test_chain_seed_changes_with_any_segment(orc):
    log_n, k, d = 7, 4, 1
    code = inputs.gen_code(log_n, 6)
    segs = inputs.gen_tables(4, 1, log_n, first_index=5)[:, 0]
    tabs = inputs.gen_tables(1, d, k, first_index=0)[0]
    _, _, f0, p0 = orc.commit_prove(code, segs, tabs, k, d, 1, 0)
    segs2 = segs.copy()
    segs2[3, 17, 0] ^= 1
    _, _, f1, p1 = orc.commit_prove(code, segs2, tabs, k, d, 1, 0)
    assert f0 != f1 and not np.array_equal(p0["challenges"], p1["challenges"])
