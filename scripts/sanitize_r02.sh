#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on the round-2 kernels (under gpurun): TMA round
# kernels (fused rounds d>=2, forced round 1), k_small (clusters, DSMEM), k_multi (TMA, in place), the
# section-4 chain (encoder + Merkle + seeded sum-check)
TAG=${1:-r02}
mkdir -p gpurun_out
cat > /tmp/san_r02.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
p = bzk.Prover(0)
# per-round kernels with TMA (k = 13, 14: two / several fused rounds), both orders, preserve + consume
for (B, d, k, order) in [(3, 2, 14, 0), (2, 3, 13, 1), (2, 2, 13, 1), (2, 4, 13, 0)]:
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 0, "adversarial")
    p.prove(t, k, d, order, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.prove(t, k, d, order)
# k_small (cluster of 2..8 CTAs)
for (B, d, k, order) in [(4, 2, 12, 0), (3, 3, 11, 1), (2, 1, 13, 0)]:
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 0, "uniform")
    p.prove(t, k, d, order, flags=bzk.BZK_F_PRESERVE_INPUT)
# k_multi (given challenges, d = 1), MSB (TMA, in place) and LSB
for order in (0, 1):
    B, k = 4, 15
    t = torch.empty((B, 1, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, 1, k, 0, "uniform")
    out = bzk.Prover.alloc_outputs(B, k, 1)
    g = torch.empty((B, 1, 16, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(g, B, 1, 4, 0, "uniform")
    out["challenges"].copy_(g[:, 0, :k])
    b = p.batch(t, k, 1, order, None, 0, bzk.BZK_F_GIVEN_CHALLENGES, out)
    bzk.bzk_prove(p.ctx, b)
torch.cuda.synchronize()
# the section-4 chain
code = inputs.gen_code(8, 6)
enc = bzk.Encoder(code, 0)
S, B, n = 4, 2, 256
codes = torch.zeros((B, S, 2 * n, 4), dtype=torch.int64, device="cuda")
codes[:, :, :n] = torch.from_numpy(inputs.gen_tables(B * S, 1, 8)[:, 0].view(np.int64).reshape(B, S, n, 4)).cuda()
roots = torch.empty((B, S, 32), dtype=torch.uint8, device="cuda")
fin = torch.empty((B, 32), dtype=torch.uint8, device="cuda")
t = torch.empty((B, 2, 1 << 11, 4), dtype=torch.int64, device="cuda")
bzk.bzk_generate(t, B, 2, 11, 0, "uniform")
out = bzk.Prover.alloc_outputs(B, 11, 2)
c = bzk.bzk_commit(S, 0, codes.data_ptr(), roots.data_ptr(), None, fin.data_ptr())
sb = bzk.make_batch(11, 2, 0, 0, B, 0, None, t, 0, 0, out["round_evals"], out["challenges"], out["final_evals"], out["claims"])
bzk.bzk_commit_prove(enc.ctx, enc.enc, c, sb)
torch.cuda.synchronize()
print("sanitizer case done")
PY
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 7 python /tmp/san_r02.py > gpurun_out/sanitize_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_${tool}_$TAG.log
done
BZK_TMA=1 timeout 1500 compute-sanitizer --tool racecheck --error-exitcode 7 python /tmp/san_r02.py > gpurun_out/sanitize_racecheck_tma1_$TAG.log 2>&1; echo "racecheck tma1 rc=$?"; tail -2 gpurun_out/sanitize_racecheck_tma1_$TAG.log
