#!/bin/bash
# ncu of k_round1_tc (c2 round 1: 1024 proofs, h = 2^19 pairs)
mkdir -p gpurun_out
TAG=${1:-r02r1}
ncu --set full --clock-control none --import-source on -k regex:k_round1_tc -c 1 -o gpurun_out/prof_r1tc_$TAG \
    python bench.py --config c2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_r1tc_$TAG.log 2>&1
ls -la gpurun_out/prof_r1tc_$TAG.ncu-rep
