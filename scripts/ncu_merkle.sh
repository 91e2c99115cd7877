#!/bin/bash
# ncu of the Merkle stage kernel (under gpurun): full set on stage 0 + launch list of one bench step
TAG=${1:-mk}; shift
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:k_merkle_stage -s 0 -c 1 \
    -o gpurun_out/prof_merkle_$TAG python bench.py --config mk20 --steps 1 --warmup 0 --no-e2e --no-cpu --batch 64 "$@" > gpurun_out/ncu_merkle_$TAG.log 2>&1
tail -2 gpurun_out/ncu_merkle_$TAG.log
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_merkle_$TAG.csv \
    python bench.py --config mk20 --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
