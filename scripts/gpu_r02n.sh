#!/bin/bash
TAG=${1:-r02n}
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 1 -o gpurun_out/prof_r1_notma_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_r1a_$TAG.log 2>&1; tail -1 gpurun_out/ncu_r1a_$TAG.log
BZK_TMA=1 ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 1 -o gpurun_out/prof_r1_tma_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_r1b_$TAG.log 2>&1; tail -1 gpurun_out/ncu_r1b_$TAG.log
