#!/bin/bash
# usage (under gpurun): bash scripts/gpu_round.sh <tag>
TAG=${1:-r01}
mkdir -p gpurun_out
python scripts/microbench.py > gpurun_out/micro_$TAG.json 2>&1
timeout 900 python -m pytest tests/ -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
for c in c3 m0 c4 c1; do
  python bench.py --config $c --steps 3 --warmup 2 --no-e2e > gpurun_out/bench_${c}_$TAG.json 2> gpurun_out/bench_${c}_$TAG.err
  cat gpurun_out/bench_${c}_$TAG.json; tail -2 gpurun_out/bench_${c}_$TAG.err
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_bench_$TAG.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 2 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_full_$TAG.log 2>&1
ls gpurun_out | head -50
