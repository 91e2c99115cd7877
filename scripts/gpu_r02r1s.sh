#!/bin/bash
# k_round1_tc launch-shape sweep (BZK_R1_CFG): parity spot check + c2 bench
TAG=${1:-r02r1s}
mkdir -p gpurun_out
for cfg in 0 1 2 3; do
  BZK_R1_CFG=$cfg ORDER=0 timeout 120 python scripts/debug_r1.py 2>&1 | grep -c "ratio g0 1\|onehot want \['0x0', '0x15', '0x54'\] got \['0x0', '0x15', '0x54'\]" | sed "s/^/cfg $cfg parity-ok: /"
  BZK_R1_CFG=$cfg timeout 180 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_r1cfg${cfg}_$TAG.json 2> gpurun_out/bench_c2_r1cfg${cfg}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_c2_r1cfg${cfg}_$TAG.json'));print('cfg $cfg', d['value'], d['kernel_ms_per_step'], d['golden_check']['mismatches'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/bench_c2_r1cfg${cfg}_$TAG.err
done
