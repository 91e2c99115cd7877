#!/bin/bash
# full evidence run: tests, smoke, every bench line, launch lists, ncu full of the top kernel, traffic captures
TAG=${1:-r01}
bash scripts/gpu_round2.sh $TAG
python bench.py --config enc20 --steps 5 --warmup 3 > gpurun_out/bench_enc20_$TAG.json 2> gpurun_out/bench_enc20_$TAG.err; cut -c1-300 gpurun_out/bench_enc20_$TAG.json
bash scripts/ncu_traffic2.sh > /dev/null 2>&1
ls gpurun_out/traffic2_* | wc -l
