#!/bin/bash
# k_multi_tc launch-shape sweep (BZK_TC_CFG, csrc/k_multi.cu BZK_TC_SHAPES): parity spot check + m0lit
TAG=${1:-r02tcs}
mkdir -p gpurun_out
for cfg in 0 1 2 3 4 5; do
  BZK_TC_CFG=$cfg timeout 300 python scripts/debug_tc.py 16,2,0 17,1,1 2>&1 | grep -c "bad rounds \[\] zero \[\] final ok True" | sed "s/^/cfg $cfg parity-ok-proofs: /"
  BZK_TC_CFG=$cfg timeout 600 python bench.py --config m0lit --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_cfg${cfg}_$TAG.json 2> gpurun_out/bench_m0lit_cfg${cfg}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_m0lit_cfg${cfg}_$TAG.json'));print('cfg $cfg', d['value'], d['kernel_ms_per_step'], d['roofline']['frac'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/bench_m0lit_cfg${cfg}_$TAG.err
done
