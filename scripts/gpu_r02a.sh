#!/bin/bash
# round-2 check: new API/full-range tests first, then the whole GPU suite, smoke, c2 bench line
TAG=${1:-r02a}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_fullrange.py -m gpu -q -x > gpurun_out/pytest_new_$TAG.log 2>&1; tail -15 gpurun_out/pytest_new_$TAG.log
timeout 1500 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -15 gpurun_out/pytest_gpu_$TAG.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?; tail -2 gpurun_out/smoke_$TAG.log
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err; cat gpurun_out/bench_c2_$TAG.json | head -c 3000; tail -3 gpurun_out/bench_c2_$TAG.err
