#!/bin/bash
# Encoder (NEXT-4) on the GPU: parity tests, bench line, size sweep.
TAG=${1:-enc}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_encoder.py -x -q > gpurun_out/pytest_enc_$TAG.log 2>&1; tail -3 gpurun_out/pytest_enc_$TAG.log
python bench.py --config enc20 --steps 5 --warmup 3 > gpurun_out/bench_enc20_$TAG.json 2> gpurun_out/bench_enc20_$TAG.err
cut -c1-1500 gpurun_out/bench_enc20_$TAG.json; tail -3 gpurun_out/bench_enc20_$TAG.err
