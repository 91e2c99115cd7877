#!/bin/bash
# full GPU suite on the current build, chain bench, c1 latency breakdown
TAG=${1:-r02e}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_chain.py tests/test_gpu_api.py -m gpu -q > gpurun_out/pytest_chain_api_$TAG.log 2>&1; tail -15 gpurun_out/pytest_chain_api_$TAG.log
timeout 1800 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -8 gpurun_out/pytest_gpu_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d['roofline'];print(sys.argv[2], d['value'], d['ms_per_step'], d['kernel_ms_per_step'], r['bound'], r['frac'], r['kernel'], d['clocks'])" $1 $2 || tail -4 ${1%.json}.err; }
timeout 600 python bench.py --config zk20 --steps 5 --warmup 3 > gpurun_out/bench_zk20_$TAG.json 2>gpurun_out/bench_zk20_$TAG.err; summ gpurun_out/bench_zk20_$TAG.json zk20
timeout 600 python bench.py --config c1 --steps 200 --warmup 20 --no-e2e --no-cpu > gpurun_out/bench_c1_$TAG.json 2>gpurun_out/bench_c1_$TAG.err; summ gpurun_out/bench_c1_$TAG.json c1
