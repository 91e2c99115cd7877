#!/bin/bash
# usage (under gpurun): bash scripts/gpu_round.sh <tag>
TAG=${1:-r01}
mkdir -p gpurun_out
python scripts/microbench.py > gpurun_out/micro_$TAG.json 2>&1
python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_bench_$TAG.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 2 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_full_$TAG.log 2>&1
ls -la gpurun_out
