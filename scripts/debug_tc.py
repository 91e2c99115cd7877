"""k_multi_tc bring-up: which rounds of a known-challenge proof differ from the oracle."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, "tests")
sys.path.insert(0, ".")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
from test_gpu_multiround import challenges, run, np64

oracle.build()
orc = oracle
cases = [tuple(int(x) for x in c.split(",")) for c in sys.argv[1:]]
for k, B, order in cases:
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 300 + k, "uniform")
    r = challenges(orc, B, k, k)
    p = bzk.Prover(0)
    out = run(p, t, k, order, r, first_index=300 + k, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.close()
    host = np64(t)
    for b in range(min(B, 2)):
        ref = orc.prove_given(host[b], k, 1, order, r[b])
        ev = np64(out["round_evals"][b]).reshape(ref["round_evals"].shape)
        bad = [i for i in range(k) if not np.array_equal(ev[i], ref["round_evals"][i])]
        zero = [i for i in range(k) if not ev[i].any()]
        fin = np.array_equal(np64(out["final_evals"][b]).reshape(ref["final_evals"].shape), ref["final_evals"])
        print(f"ctas={os.environ.get('BZK_TC_CTAS')} k={k} B={B} order={order} b={b}: bad rounds {bad} zero {zero} final ok {fin}", flush=True)

# value-level look at one failing proof
if os.environ.get("DETAIL"):
    k, B, order = 16, 1, 1
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 300 + k, "uniform")
    r = challenges(orc, B, k, k)
    p = bzk.Prover(0)
    out = run(p, t, k, order, r, first_index=300 + k, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.close()
    host = np64(t)
    ref = orc.prove_given(host[0], k, 1, order, r[0])
    P = int.from_bytes(b"".join(x.to_bytes(8, "little") for x in inputs.P_BN254), "little")
    ev = np64(out["round_evals"][0]).reshape(ref["round_evals"].shape)
    val = lambda a: int.from_bytes(a.astype("<u8").tobytes(), "little")
    R = pow(2, 256, P)
    for i in range(k):
        g, w = [val(ev[i][j]) for j in range(2)], [val(ref["round_evals"][i][j]) for j in range(2)]
        print(i, [hex(x)[:18] for x in g], [hex(x)[:18] for x in w], "ratio", [(gg * pow(ww, -1, P)) % P if ww else None for gg, ww in zip(g, w)][:1])
    print("claim", hex(val(np64(out["claims"][0])))[:18], hex(val(ref["claims"]))[:18])
