#!/bin/bash
# d = 3 round 1 with unreduced 512-bit products in the fused rounds too: parity,
# c3, launch list
TAG=${1:-r02w3f}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_d3_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_q3_$TAG.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_q3_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
timeout 900 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_c3_$TAG.json 2> gpurun_out/bench_c3_$TAG.err; summ gpurun_out/bench_c3_$TAG.json c3
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_$TAG.csv \
    python bench.py --config c3 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/launches_c3_$TAG.csv | grep -v "generate\|init_consts"
