#!/bin/bash
# k_round1_tc bring-up: parity, smoke, c2 with and without the tensor-core round 1
TAG=${1:-r02r1}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_round1_tc.py -x -q > gpurun_out/pytest_r1_$TAG.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_r1_$TAG.log
for r1 in 1 0; do
  BZK_R1_TC=$r1 timeout 180 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_r1tc${r1}_$TAG.json 2> gpurun_out/bench_c2_r1tc${r1}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_c2_r1tc${r1}_$TAG.json'));print('r1tc=$r1', d['value'], d['kernel_ms_per_step'], d['golden_check'], d['clocks']['sm_mhz'])" || tail -5 gpurun_out/bench_c2_r1tc${r1}_$TAG.err
done
