#!/bin/bash
TAG=${1:-x}
python bench.py --config g2 > gpurun_out/bench_g2_$TAG.json 2>&1; cat gpurun_out/bench_g2_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_g2_$TAG.csv \
    python bench.py --config g2 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_gl_round -s 0 -c 2 \
    -o gpurun_out/prof_g2_$TAG python bench.py --config g2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_g2_$TAG.log 2>&1
tail -1 gpurun_out/ncu_g2_$TAG.log
