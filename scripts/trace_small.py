"""Phase timing of k_small rounds (instrumented build libbzk_trace.so; not part of the product)."""
import os, sys
os.environ["BZK_LIB"] = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "paper_conf_asplos_lucw0cz25_b200", "libbzk_trace.so")
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np, torch
from paper_conf_asplos_lucw0cz25_b200 import bzk
B, d, k = 16, 2, 12
t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
bzk.bzk_generate(t, B, d, k, 0, "uniform")
out = bzk.Prover.alloc_outputs(B, k, d)
big = torch.zeros((B + 400, 4), dtype=torch.int64, device="cuda")
out["claims"] = big
p = bzk.Prover(0)
for _ in range(3):
    p.prove(t, k, d, 0, flags=bzk.BZK_F_PRESERVE_INPUT, out=out)
torch.cuda.synchronize()
raw = big.cpu().numpy().reshape(-1).view(np.int64)
T = raw[15 * 4:15 * 4 + 1000].reshape(-1, 10)
names = ["eval+warpreduce", "sync1", "gather(leader warp)", "load st", "sha256 x3", "stores", "r R", "sync2", "fold+next eval"]
for r in range(1, 9):
    row = T[r]
    print(r, " ".join(f"{n}={row[i+1]-row[i]}" for i, n in enumerate(names)), "total", row[9] - row[0])
