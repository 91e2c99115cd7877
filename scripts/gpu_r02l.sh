#!/bin/bash
TAG=${1:-r02l}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api.py tests/test_gpu_multiround.py tests/test_gpu_chain.py tests/test_gpu_fullrange.py -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -2 gpurun_out/pytest_gpu_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], d.get('kernel_ms_per_step'), r.get('bound'), r.get('frac'), r.get('kernel'), d['clocks'])" $1 $2 || tail -4 ${1%.json}.err; }
for v in "BZK_SMALL=0" "BZK_SMALL=1"; do
  env $v timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_${v}_$TAG.json 2>gpurun_out/bench_c1_${v}_$TAG.err; summ gpurun_out/bench_c1_${v}_$TAG.json "c1 $v"
done
