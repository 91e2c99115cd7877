"""Writes tests/golden/proof_small.txt using ONLY oracle/ (never the CUDA path).

    python tests/golden/make_golden.py

Each case's tables come from paper_conf_asplos_lucw0cz25_b200.inputs (counter-based
generator, no method arithmetic); the transcript seed is inputs.DEFAULT_SEED.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_asplos_lucw0cz25_b200 import inputs  # noqa: E402

# (k, d, order, index, dist): uniform is over the whole field [0, p); adversarial reaches p - 1,
# [p - 2^16, p), alternating 0 / p - 1 and [2^253, ...) (inputs.py)
CASES = [(4, 2, 0, 0, "uniform"), (4, 2, 1, 1, "uniform"), (3, 3, 0, 5, "uniform"), (5, 1, 1, 2, "uniform"),
         (2, 4, 0, 3, "uniform"), (4, 2, 0, 20, "adversarial"), (5, 3, 1, 21, "adversarial"),
         (3, 4, 0, 22, "adversarial"), (6, 1, 1, 23, "adversarial")]


def main():
    lines = ["# Frozen oracle output (SURVEY.md 8(c.2) transcript reading, DESIGN.md R5-R7).",
             "# Written by tests/golden/make_golden.py from oracle/ only.",
             "# case k d order index, then rows: <key> <hex values...>"]
    for k, d, order, I, dist in CASES:
        t = inputs.gen_tables(1, d, k, first_index=I, dist=dist)[0]
        out = oracle.prove(t, k, d, order, inputs.DEFAULT_SEED, I)
        lines.append(f"case k={k} d={d} order={order} index={I} dist={dist}")
        for key in ("round_evals", "challenges", "final_evals", "claims"):
            vals = oracle.from_limbs(out[key])
            lines.append(key + " " + " ".join(f"{v:x}" for v in vals))
    with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "proof_small.txt"), "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
