#!/bin/bash
# k_small (single-launch cluster proofs): parity (full suite), c1 latency A/B, c4 A/B
TAG=${1:-r02h}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/ -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -4 gpurun_out/pytest_gpu_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], d.get('kernel_ms_per_step'), r.get('bound'), r.get('frac'), r.get('kernel'), d['clocks'])" $1 $2 || tail -4 ${1%.json}.err; }
for v in "BZK_SMALL=0" "BZK_SMALL=1"; do
  env $v timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_${v}_$TAG.json 2>gpurun_out/bench_c1_${v}_$TAG.err; summ gpurun_out/bench_c1_${v}_$TAG.json "c1 $v"
  env $v timeout 600 python bench.py --config c4 --steps 5 --warmup 3 > gpurun_out/bench_c4_${v}_$TAG.json 2>gpurun_out/bench_c4_${v}_$TAG.err; python -c "import json;d=json.load(open('gpurun_out/bench_c4_${v}_$TAG.json'));print('c4 $v', d['value'], d['overlap'])"
done
