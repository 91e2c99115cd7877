#!/bin/bash
# ncu of the encoder (under gpurun): launch list of one bench step + full set on the first A_0 and B_0 launches
TAG=${1:-enc}; shift
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_enc_$TAG.csv \
    python bench.py --config enc20 --steps 1 --warmup 0 --no-e2e --no-cpu --batch 64 "$@" > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_spmv -s 0 -c 1 \
    -o gpurun_out/prof_enc_A0_$TAG python bench.py --config enc20 --steps 1 --warmup 0 --no-e2e --no-cpu --batch 64 "$@" > gpurun_out/ncu_enc_$TAG.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_spmv -s 14 -c 1 \
    -o gpurun_out/prof_enc_B0_$TAG python bench.py --config enc20 --steps 1 --warmup 0 --no-e2e --no-cpu --batch 64 "$@" >> gpurun_out/ncu_enc_$TAG.log 2>&1
tail -2 gpurun_out/ncu_enc_$TAG.log
