"""Host logic of bench.py (-m "not gpu"): the algorithmic-work formulas behind every roofline number."""
import importlib.util
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def load_bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    argv = sys.argv
    sys.argv = ["bench.py"]
    try:
        spec.loader.exec_module(m)
    finally:
        sys.argv = argv
    return m


def test_alg_mulmods_total_is_sum_over_rounds():
    b = load_bench()
    for d in (1, 2, 3, 4):
        for k in (12, 20, 22):
            # per round i (h = 2^(k-i) pairs): d folds of round i-1's pairs (2h products) + the
            # evaluation products; the total of the method is d^2 (2^k - 1)
            assert b.alg_mulmods(d, k, "total") == d * d * ((1 << k) - 1)
            tail_log = 8
            i0 = k - tail_log
            fused = sum(2 * d * (1 << (k - i)) + d * (d - 1) * (1 << (k - i)) for i in range(2, i0))
            assert b.alg_mulmods(d, k, "fused") == fused
            assert b.alg_mulmods(d, k, "round1") == (d + 1) * (d - 1) * (1 << (k - 1))


def test_alg_bytes_per_kind():
    b = load_bench()
    d, k = 2, 20
    assert b.alg_bytes_kind(d, k, "round1") == d * (1 << k) * 32
    # fused round i reads 4 d h and writes 2 d h elements
    assert b.alg_bytes_kind(d, k, "fused") == sum(6 * d * (1 << (k - i)) * 32 for i in range(2, k - 8))
    assert b.alg_bytes_kind(d, k, "fused", esz=8) * 4 == b.alg_bytes_kind(d, k, "fused")


def test_sha256_alu_only_instruction_count():
    b = load_bench()
    # 64 rounds x (6 rotations + 4 three-input logic ops) + 48 schedule steps x (6 shifts/rotations + 2 xors)
    assert b.ALU_OPS_PER_COMPRESSION == 64 * (6 + 4) + 48 * (6 + 2) == 1024


def test_encoder_edge_count():
    b = load_bench()
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    code = inputs.gen_code(10, 6)
    n = 1 << 10
    # levels 0, 1: A_l has c n_l edges, B_l has d n_l / 2; base G0 dense 64 x 64
    exp = sum(inputs.ENC_C * (n >> (2 * l)) + inputs.ENC_D * (n >> (2 * l)) // 2 for l in range(2)) + 64 * 64
    assert b.enc_edges(code) == exp
