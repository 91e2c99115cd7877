#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small configurations (under gpurun)
TAG=${1:-x}
mkdir -p gpurun_out
cat > /tmp/san_case.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_asplos_lucw0cz25_b200 import bzk
p = bzk.Prover(0)
for (B, d, k, order) in [(4, 2, 12, 0), (3, 3, 11, 1), (2, 1, 14, 0), (2, 4, 9, 1)]:
    t = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(t, B, d, k, 0, "uniform")
    p.prove(t, k, d, order, flags=bzk.BZK_F_PRESERVE_INPUT)
    p.prove(t, k, d, order)      # consume mode
torch.cuda.synchronize()
print("sanitizer case done")
PY
for tool in memcheck racecheck synccheck; do
  compute-sanitizer --tool $tool --error-exitcode 7 python /tmp/san_case.py > gpurun_out/sanitize_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_${tool}_$TAG.log
done
