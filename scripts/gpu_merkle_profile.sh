#!/bin/bash
# Merkle (NEXT-3) evidence run: parity, bench lines (both modes), Table 3 size sweep, launch list, ncu full.
TAG=${1:-mk}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_merkle.py -x -q > gpurun_out/pytest_merkle_$TAG.log 2>&1; tail -2 gpurun_out/pytest_merkle_$TAG.log
for c in mk20 mk20f; do
  python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/bench_${c}_$TAG.json 2> gpurun_out/bench_${c}_$TAG.err
  cut -c1-300 gpurun_out/bench_${c}_$TAG.json; tail -2 gpurun_out/bench_${c}_$TAG.err
done
# paper Table 3 sizes (2^18..2^22 blocks per tree), 16 GiB of blocks per step
for n in 18 19 20 21 22; do
  B=$(( 256 << (20 - n) )); [ $n -gt 20 ] && B=$(( 256 >> (n - 20) ))
  python bench.py --config mk20 --log-blocks $n --batch $B --steps 5 --warmup 3 --no-e2e --no-cpu >> gpurun_out/merkle_sizes_$TAG.jsonl 2>/dev/null
done
python bench.py --config mk20 --impl reference --steps 1 --warmup 3 > gpurun_out/bench_mk20_ref_$TAG.json 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_merkle_$TAG.csv \
    python bench.py --config mk20 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_merkle_stage -s 0 -c 1 \
    -o gpurun_out/prof_merkle_$TAG python bench.py --config mk20 --steps 1 --warmup 0 --no-e2e --no-cpu --batch 64 > gpurun_out/ncu_merkle_$TAG.log 2>&1
tail -1 gpurun_out/ncu_merkle_$TAG.log
