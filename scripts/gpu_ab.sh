#!/bin/bash
# A/B run: parity suite on the main library, then bench lines of variant libraries / env knobs.
# usage (under gpurun): bash scripts/gpu_ab.sh <tag> "LABEL:ENV..." ...
TAG=${1:-x}; shift
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/ -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
for spec in "$@"; do
  label=${spec%%:*}; envs=${spec#*:}
  echo "== $label ($envs)"
  env $envs python bench.py --no-e2e --no-cpu --steps 3 --warmup 3 ${BENCH_ARGS} > gpurun_out/ab_${TAG}_$label.json 2> gpurun_out/ab_${TAG}_$label.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'], d['clocks'])" gpurun_out/ab_${TAG}_$label.json || tail -3 gpurun_out/ab_${TAG}_$label.err
done
