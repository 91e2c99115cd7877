"""Writes tests/golden/merkle_small.txt using ONLY oracle/ (never the CUDA path).

    python tests/golden/make_golden_merkle.py

Blocks come from paper_conf_asplos_lucw0cz25_b200.inputs.gen_blocks (counter-based generator,
no hashing).  Rows: n mode tree_index root_hex (mode 0 = one SHA-256 compression per 512-bit
block, mode 1 = FIPS SHA-256; readings R17-R19).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_asplos_lucw0cz25_b200 import inputs  # noqa: E402

CASES = [(0, 0, 0), (0, 1, 0), (1, 0, 1), (3, 0, 2), (3, 1, 2), (6, 0, 3), (6, 1, 4), (10, 0, 5), (10, 1, 5)]


def main():
    lines = ["# Frozen Merkle roots from oracle/ (DESIGN.md R17-R19), written by make_golden_merkle.py.",
             "# n mode tree_index root_hex"]
    for n, mode, idx in CASES:
        root, _ = oracle.merkle(inputs.gen_blocks(1, n, first_index=idx)[0], n, mode, nodes=False)
        lines.append(f"{n} {mode} {idx} {root.hex()}")
    with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "merkle_small.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
