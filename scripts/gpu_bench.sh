#!/bin/bash
# One gpurun call: GPU tests, bench line, ncu launch list and one full ncu capture of the top kernel.
# usage (under gpurun): bash scripts/gpu_bench.sh <tag> [bench args...]
set -x
TAG=${1:-r01}; shift
mkdir -p gpurun_out
python bench.py "$@" > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -3 gpurun_out/bench_$TAG.err
cat gpurun_out/bench_$TAG.json
