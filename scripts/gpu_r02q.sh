#!/bin/bash
TAG=${1:-r02q}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_encoder.py tests/test_gpu_chain.py -m gpu -q -x > gpurun_out/pytest_q_$TAG.log 2>&1; tail -2 gpurun_out/pytest_q_$TAG.log
for cfg in enc20 zk20; do
  timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_$TAG.json 2> gpurun_out/bench_${cfg}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_${cfg}_$TAG.json'));print('$cfg', d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'], d['clocks'])" || tail -3 gpurun_out/bench_${cfg}_$TAG.err
done
