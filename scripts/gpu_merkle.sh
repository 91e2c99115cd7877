#!/bin/bash
# Merkle module (NEXT-3) on the GPU: parity tests, bench lines of both hash modes, A/B of variants.
# usage: bash scripts/gpu_merkle.sh TAG [LABEL:ENV ...]   (ENV e.g. BZK_LIB=...libbzk_fma.so,BZK_MK_LT=4)
TAG=${1:-mk}; shift
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_merkle.py -x -q > gpurun_out/pytest_merkle_$TAG.log 2>&1; tail -3 gpurun_out/pytest_merkle_$TAG.log
for c in mk20 mk20f; do
  python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_${c}_$TAG.json 2> gpurun_out/bench_${c}_$TAG.err
  cut -c1-400 gpurun_out/bench_${c}_$TAG.json; tail -2 gpurun_out/bench_${c}_$TAG.err
done
for spec in "$@"; do
  label=${spec%%:*}; envs=${spec#*:}
  env ${envs//,/ } python bench.py --config mk20 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_mk_${TAG}_$label.json 2>&1
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['ms_per_step'], d['roofline']['achieved'], d['roofline']['frac'], d['clocks']['sm_mhz'])" gpurun_out/ab_mk_${TAG}_$label.json $label || tail -3 gpurun_out/ab_mk_${TAG}_$label.json
done
