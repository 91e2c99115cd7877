#!/bin/bash
# bench lines with the per-kernel HBM roofline (c2 default, c3, g2, m0lit, c1)
TAG=${1:-r02pk}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_c2_$TAG.json'));print('c2', d['value'], d['clocks']['sm_mhz'], json.dumps(d['roofline'].get('per_kernel_hbm')))" || tail -5 gpurun_out/bench_c2_$TAG.err
for cfg in c3 g2 m0lit; do
  timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_$TAG.json 2> gpurun_out/bench_${cfg}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_${cfg}_$TAG.json'));print('$cfg', d['value'], json.dumps(d['roofline'].get('per_kernel_hbm')))" || tail -5 gpurun_out/bench_${cfg}_$TAG.err
done
timeout 600 python bench.py --config c1 --steps 500 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_$TAG.json 2> gpurun_out/bench_c1_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_c1_$TAG.json'));print('c1', d['value'])" || tail -5 gpurun_out/bench_c1_$TAG.err
