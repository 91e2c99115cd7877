#!/bin/bash
TAG=${1:-r02i}
mkdir -p gpurun_out
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], d.get('kernel_ms_per_step'), r.get('bound'), r.get('frac'), r.get('kernel'), d['clocks'])" $1 $2 || tail -4 ${1%.json}.err; }
for v in "BZK_SMALL=0" "BZK_SMALL=1"; do
  env $v timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_${v}_$TAG.json 2>gpurun_out/bench_c1_${v}_$TAG.err; summ gpurun_out/bench_c1_${v}_$TAG.json "c1 $v"
done
env BZK_SMALL=1 timeout 600 python bench.py --config c4 --steps 5 --warmup 3 > gpurun_out/bench_c4_$TAG.json 2>gpurun_out/bench_c4_$TAG.err; python -c "import json;d=json.load(open('gpurun_out/bench_c4_$TAG.json'));print('c4', d['value'], d['overlap'])"
ncu --set full --clock-control none --import-source on -k regex:k_small -s 5 -c 1 -o gpurun_out/prof_c1_small_$TAG python bench.py --config c1 --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/ncu_c1_$TAG.log 2>&1; tail -1 gpurun_out/ncu_c1_$TAG.log
