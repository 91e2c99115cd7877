#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small Merkle (NEXT-3), encoder (NEXT-4) and
# Goldilocks (NEXT-2) cases (under gpurun)
TAG=${1:-x}
mkdir -p gpurun_out
cat > /tmp/san_mod.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
import torch
from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
mb = bzk.MerkleBuilder(0)
for n, B, mode in [(0, 2, 0), (3, 3, 1), (9, 2, 0), (12, 2, 1)]:
    blocks = torch.empty((B, 1 << n, 64), dtype=torch.uint8, device="cuda")
    bzk.bzk_generate_blocks(blocks, B, n, 0)
    mb.build(blocks, n, mode)
    mb.build(blocks, n, mode, with_nodes=False)
code = inputs.gen_code(10, 6)
enc = bzk.Encoder(code, ctx=mb.ctx)
m = inputs.gen_tables(3, 1, 10)[:, 0]
c = torch.zeros((3, 2048, 4), dtype=torch.int64, device="cuda")
c[:, :1024] = torch.from_numpy(m.view(np.int64)).cuda()
enc.encode(c)
p = bzk.Prover(0)
t = torch.empty((2, 2, 1 << 11), dtype=torch.int64, device="cuda")
bzk.bzk_generate(t, 2, 2, 11, 0, "gl")
p.prove(t, 11, 2, 0, flags=bzk.BZK_F_FIELD_GOLDILOCKS | bzk.BZK_F_PRESERVE_INPUT)
torch.cuda.synchronize()
enc.close()
print("sanitizer module case done")
PY
for tool in memcheck racecheck synccheck; do
  compute-sanitizer --tool $tool --error-exitcode 7 python /tmp/san_mod.py > gpurun_out/sanitize_mod_${tool}_$TAG.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_mod_${tool}_$TAG.log
done
