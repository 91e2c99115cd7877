#!/bin/bash
# ncu of k_multi_tc (m0lit pass 1: 1024 proofs, K = 20) + the launch list and DRAM bytes of every pass
mkdir -p gpurun_out
TAG=${1:-r02tc}
ncu --set full --clock-control none --import-source on -k regex:k_multi_tc -c 1 -o gpurun_out/prof_multi_tc_$TAG \
    python bench.py --config m0lit --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_multi_tc_$TAG.log 2>&1
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:"k_multi|k_tail|k_transcript" --csv python bench.py --config m0lit --steps 1 --warmup 0 --no-e2e --no-cpu \
    > gpurun_out/traffic_m0lit_$TAG.csv 2>/dev/null
ls -la gpurun_out/prof_multi_tc_$TAG.ncu-rep gpurun_out/traffic_m0lit_$TAG.csv
