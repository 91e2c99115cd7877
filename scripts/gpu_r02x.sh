#!/bin/bash
# launch-shape sweep with the TMA fused rounds (pairs-per-thread cap, CTA waves)
TAG=${1:-r02x}
mkdir -p gpurun_out
for v in "BZK_PPT_MAX=256" "BZK_PPT_MAX=64" "BZK_PPT_MAX=1024" "BZK_CTA_WAVES=2" "BZK_CTA_WAVES=8" "BZK_PPT_MAX=256"; do
  env $v timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw.json 2> gpurun_out/sw.err
  python -c "import json;d=json.load(open('gpurun_out/sw.json'));print('$v', d['value'], d['kernel_ms_per_step'], d['clocks']['sm_mhz'])" || tail -2 gpurun_out/sw.err
done
