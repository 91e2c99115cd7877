#!/bin/bash
TAG=${1:-r02t}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullrange.py -m gpu -q -x -k "sweep or config or sha256 or given" > gpurun_out/pytest_t_$TAG.log 2>&1; tail -2 gpurun_out/pytest_t_$TAG.log
for v in "BZK_SMALL=0" "BZK_SMALL=1"; do
  env $v timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_${v}_$TAG.json 2>gpurun_out/bench_c1_${v}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_c1_${v}_$TAG.json'));print('c1 $v', d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['clocks'])"
done
