#!/bin/bash
# Table 4 analogue: m0 (Fiat-Shamir) and m0lit (given challenges) at k = 18..22, d = 1, MSB
TAG=${1:-r02s}
mkdir -p gpurun_out
: > gpurun_out/sizes_m0_$TAG.jsonl
for cfg in m0 m0lit; do
  for k in 18 19 20 21 22; do
    B=1024; [ $k -ge 22 ] && B=512
    timeout 900 python bench.py --config $cfg --k $k --batch $B --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/tmp.json 2> gpurun_out/tmp.err && cat gpurun_out/tmp.json >> gpurun_out/sizes_m0_$TAG.jsonl
    python -c "import json;d=json.load(open('gpurun_out/tmp.json'));print('$cfg k=$k B=$B', d['value'], d['roofline']['bound'], d['roofline']['frac'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/tmp.err
  done
done
