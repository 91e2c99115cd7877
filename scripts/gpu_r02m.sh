#!/bin/bash
TAG=${1:-r02m}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_chain.py -m gpu -q -x > gpurun_out/pytest_chain_$TAG.log 2>&1; tail -2 gpurun_out/pytest_chain_$TAG.log
for v in 1 2 4 8; do
  BZK_CHAIN_CHUNKS=$v timeout 600 python bench.py --config zk20 --steps 5 --warmup 3 > gpurun_out/bench_zk20_ch${v}_$TAG.json 2>gpurun_out/bench_zk20_ch${v}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_zk20_ch${v}_$TAG.json'));print('zk20 chunks=$v', d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['clocks'])" || tail -3 gpurun_out/bench_zk20_ch${v}_$TAG.err
done
