#!/bin/bash
# k_fused_tc<2>: tensor-core-only deltas kept unreduced (< 4p): parity, c2, launch list
TAG=${1:-r02rd}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_rd_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_rd_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for i in 1 2; do
timeout 900 python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_${i}_$TAG.json 2> gpurun_out/bench_c2_${i}_$TAG.err; summ gpurun_out/bench_c2_${i}_$TAG.json c2_$i
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/launches_c2_$TAG.csv | grep -v generate
