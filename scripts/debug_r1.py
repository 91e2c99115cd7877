"""k_round1_tc bring-up: round-1 values vs Python sums for structured inputs."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, "tests"); sys.path.insert(0, ".")
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
oracle.build()
P = oracle.P
R = pow(2, 256, P)
val = lambda a: int.from_bytes(np.ascontiguousarray(a).astype("<u8").tobytes(), "little")
np64 = lambda t: t.detach().cpu().numpy().view(np.uint64)
k = int(os.environ.get("K", "15")); order = int(os.environ.get("ORDER", "0"))
N = 1 << k
for name in ["ones_small", "uniform", "onehot"]:
    if name == "uniform":
        host = inputs.gen_tables(1, 2, k, first_index=3)
    else:
        host = np.zeros((1, 2, N, 4), dtype=np.uint64)
        if name == "ones_small":
            host[0, :, :, 0] = 1
        else:
            host[0, 0, 5, 0] = 3; host[0, 1, 5, 0] = 7   # one nonzero product at entry 5
    t = torch.from_numpy(host.view(np.int64)).cuda()
    out = bzk.Prover.alloc_outputs(1, k, 2)
    p = bzk.Prover(0)
    bzk.bzk_prove(p.ctx, p.batch(t, k, 2, order, None, 0, bzk.BZK_F_PRESERVE_INPUT, out))
    torch.cuda.synchronize(); p.close()
    ev = np64(out["round_evals"][0]).reshape(k, 3, 4)
    T0 = [val(host[0, 0, i]) for i in range(N)]; T1 = [val(host[0, 1, i]) for i in range(N)]
    h = N // 2
    if order == 0: pa = [(2 * j, 2 * j + 1) for j in range(h)]
    else: pa = [(j, j + h) for j in range(h)]
    g0 = sum(T0[a] * T1[a] for a, _ in pa) % P
    g1 = sum(T0[b] * T1[b] for _, b in pa) % P
    g2 = sum((2 * T0[b] - T0[a]) * (2 * T1[b] - T1[a]) for a, b in pa) % P
    got = [val(ev[0, i]) for i in range(3)]
    print(name, "want", [hex(x)[:14] for x in (g0, g1, g2)], "got", [hex(x)[:14] for x in got],
          "ratio g0", (got[0] * pow(g0, -1, P)) % P if g0 else None)
