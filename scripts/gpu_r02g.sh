#!/bin/bash
# after the latency changes (static-layout transcript hash, warp-parallel Lagrange, Montgomery-form tail
# tables) and the k_multi weight fix: full GPU suite, c1 latency (long run for clock samples), c2, m0lit
TAG=${1:-r02g}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/ -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -4 gpurun_out/pytest_gpu_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d['roofline'];print(sys.argv[2], d['value'], d['ms_per_step'], d['kernel_ms_per_step'], r['bound'], r['frac'], r['kernel'], d['clocks'])" $1 $2 || tail -4 ${1%.json}.err; }
timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 --no-e2e --no-cpu > gpurun_out/bench_c1_$TAG.json 2>gpurun_out/bench_c1_$TAG.err; summ gpurun_out/bench_c1_$TAG.json c1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_$TAG.json 2>gpurun_out/bench_c2_$TAG.err; summ gpurun_out/bench_c2_$TAG.json c2
timeout 600 python bench.py --config m0lit --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_$TAG.json 2>gpurun_out/bench_m0lit_$TAG.err; summ gpurun_out/bench_m0lit_$TAG.json m0lit
