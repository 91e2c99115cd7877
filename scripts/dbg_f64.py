import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import oracle
from paper_conf_asplos_lucw0cz25_b200 import bzk
P = oracle.P
vals = [(1, 1), (2, 3), (P - 1, P - 1), (2**255, 3), (12345678901234567890, 98765432109876543210), (2**48, 2**48)]
A = torch.from_numpy(oracle.to_limbs([a for a, b in vals]).view(np.int64)).cuda()
B = torch.from_numpy(oracle.to_limbs([b for a, b in vals]).view(np.int64)).cuda()
out = torch.empty_like(A)
bzk.bzk_debug_field(5, len(vals), A, B, out)
torch.cuda.synchronize()
got = oracle.from_limbs(out.cpu().numpy().view(np.uint64))
inv = pow(2**288, P - 2, P)
for (a, b), g in zip(vals, got):
    e = a * b * inv % P
    print(hex(a)[:20], hex(b)[:20], "ok" if g == e else "BAD", hex(g), hex(e), hex((g - e) % P))
