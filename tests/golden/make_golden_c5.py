"""Writes tests/golden/c5_proof_digests.txt using ONLY oracle/ (never the CUDA path).

    python tests/golden/make_golden_c5.py [--n 8192] [--procs 6]

Per-proof digests of BASELINE configs[1]/[4] (d = 2, k = 20, LSB order, uniform tables from
paper_conf_asplos_lucw0cz25_b200.inputs, transcript seed inputs.DEFAULT_SEED) for global proof
indices 0..n-1 -- the proofs bench.py's c2 (1024 per GPU, weak scaling: indices 0..1024 W - 1) and
c5 (8192 sharded by proof) runs produce.  Digest of proof I = first 8 bytes (hex) of
SHA-256(round_evals || challenges || final_evals || claim), each the little-endian u64 limbs as the
C ABI lays them out.  Resumable: proofs already in the file are skipped.
"""
import hashlib
import multiprocessing as mp
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
OUT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "c5_proof_digests.txt")
D, K, ORDER = 2, 20, 0


def proof_digest(out) -> str:
    h = hashlib.sha256()
    for key in ("round_evals", "challenges", "final_evals", "claims"):
        h.update(out[key].astype("<u8").tobytes())
    return h.hexdigest()[:16]


def one(i):
    import oracle
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    t = inputs.gen_tables(1, D, K, first_index=i)[0]
    return i, proof_digest(oracle.prove(t, K, D, ORDER, inputs.DEFAULT_SEED, i))


def main():
    n = int(sys.argv[sys.argv.index("--n") + 1]) if "--n" in sys.argv else 8192
    procs = int(sys.argv[sys.argv.index("--procs") + 1]) if "--procs" in sys.argv else 6
    import oracle
    oracle.build()
    done = {}
    if os.path.exists(OUT):
        for ln in open(OUT):
            if ln.strip() and not ln.startswith("#"):
                i, d = ln.split()
                done[int(i)] = d
    todo = [i for i in range(n) if i not in done]
    with mp.Pool(procs) as pool, open(OUT, "a") as f:
        if not done:
            f.write("# per-proof digests, d=2 k=20 LSB uniform, seed 0x00..0x1f: index sha256(outputs)[:8]\n")
            f.write("# written by tests/golden/make_golden_c5.py from oracle/ only\n")
        for i, d in pool.imap_unordered(one, todo, chunksize=4):
            f.write(f"{i} {d}\n")
            f.flush()


if __name__ == "__main__":
    main()
