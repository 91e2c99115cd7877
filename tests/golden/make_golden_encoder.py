"""Writes tests/golden/encoder_small.txt using ONLY oracle/ (never the CUDA path).

    python tests/golden/make_golden_encoder.py

Rows: log_n message_index sha256(codeword bytes, LE u64 limbs).  Graphs from inputs.gen_code(log_n, 6);
messages are inputs.gen_tables(1, 1, log_n, first_index=message_index)[0, 0] (R21-R24).
"""
import hashlib
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_asplos_lucw0cz25_b200 import inputs  # noqa: E402

CASES = [(6, 0), (7, 1), (8, 2), (11, 3)]


def main():
    lines = ["# Frozen encoder codeword digests from oracle/ (DESIGN.md R21-R24), make_golden_encoder.py.",
             "# log_n message_index sha256(codeword LE u64 limbs)"]
    for log_n, idx in CASES:
        code = inputs.gen_code(log_n, 6)
        c = oracle.encode(code, inputs.gen_tables(1, 1, log_n, first_index=idx)[0, 0])
        lines.append(f"{log_n} {idx} {hashlib.sha256(c.astype('<u8').tobytes()).hexdigest()}")
    with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "encoder_small.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
