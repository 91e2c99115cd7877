#!/bin/bash
# One gpurun call: GPU parity suite, headline bench line, launch list, DRAM traffic of the fused rounds.
# usage (under gpurun): bash scripts/gpu_check.sh <tag> [config]
TAG=${1:-x}; CFG=${2:-c2}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/ -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?; tail -2 gpurun_out/smoke_$TAG.log
python bench.py --config $CFG > gpurun_out/bench_${CFG}_$TAG.json 2> gpurun_out/bench_${CFG}_$TAG.err; cat gpurun_out/bench_${CFG}_$TAG.json; tail -3 gpurun_out/bench_${CFG}_$TAG.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}_$TAG.csv \
    python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
# DRAM bytes of every k_round launch of one step (application replay: no device-memory save/restore)
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,launch__grid_size --clock-control none \
    --replay-mode application -k regex:"k_round|k_gl_round" --csv --log-file gpurun_out/traffic_${CFG}_$TAG.csv \
    python bench.py --config $CFG --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_traffic_${CFG}_$TAG.log 2>&1
tail -2 gpurun_out/ncu_traffic_${CFG}_$TAG.log
ls gpurun_out | wc -l
