#!/bin/bash
# NEXT-1 multi-round parity + m0lit A/B (passes of 2 vs 3 rounds, vs per-round kernels), c2 with the
# TMA policy, ncu --set full of the c2 round kernels (round 1 + round 2, batch 256)
TAG=${1:-r02c}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multiround.py tests/test_gpu_parity.py -m gpu -q -x -k "multiround or given or m0lit" > gpurun_out/pytest_multi_$TAG.log 2>&1; tail -5 gpurun_out/pytest_multi_$TAG.log
for v in "BZK_MULTI=0" "BZK_MULTI_M=2" "BZK_MULTI_M=3"; do
  env $v timeout 600 python bench.py --config m0lit --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_${v}_$TAG.json 2>gpurun_out/bench_m0lit_${v}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_m0lit_${v}_$TAG.json'));print('m0lit $v', d['value'], d['kernel_ms_per_step'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/bench_m0lit_${v}_$TAG.err
done
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_$TAG.json 2>gpurun_out/bench_c2_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_c2_$TAG.json'));print('c2', d['value'], d['kernel_ms_per_step'], d['clocks'])"
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 2 \
    -o gpurun_out/prof_c2_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_full_$TAG.log 2>&1
tail -2 gpurun_out/ncu_full_$TAG.log
