#!/bin/bash
# End-of-round check of the final code: GPU suite, smoke, c2 / c3 bench lines
TAG=${1:-r02end}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -2 gpurun_out/pytest_gpu_$TAG.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/smoke_$TAG.log | cut -c1-120
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
timeout 1200 python bench.py > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err; summ gpurun_out/bench_c2_$TAG.json c2
timeout 900 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_c3_$TAG.json 2> gpurun_out/bench_c3_$TAG.err; summ gpurun_out/bench_c3_$TAG.json c3
