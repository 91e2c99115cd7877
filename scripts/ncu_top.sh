#!/bin/bash
# usage (under gpurun): bash scripts/ncu_top.sh <tag> [extra bench args]
TAG=${1:-x}; shift
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 2 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 "$@" > gpurun_out/ncu_full_$TAG.log 2>&1
tail -2 gpurun_out/ncu_full_$TAG.log
