#!/bin/bash
# DRAM traffic of every fused-round launch of one bench step at the bench configuration (under gpurun)
TAG=${1:-x}
ncu --set full --clock-control none -k regex:"k_round" -c 11 -o gpurun_out/traffic_$TAG \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_traffic_$TAG.log 2>&1
ncu -i gpurun_out/traffic_$TAG.ncu-rep --page raw --csv --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,launch__grid_size > gpurun_out/traffic_$TAG.csv 2>&1
