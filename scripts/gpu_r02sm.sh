#!/bin/bash
# 2-warp k_fused_tc for the late d = 2 rounds: parity (incl. forced on / off), c2, c2 launch list
TAG=${1:-r02sm}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_sm_$TAG.log 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/pytest_sm_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in 12 0; do
BZK_FTC_SMALL_LOG=$v timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_sm${v}_$TAG.json 2> gpurun_out/bench_c2_sm${v}_$TAG.err; summ gpurun_out/bench_c2_sm${v}_$TAG.json c2_sm$v
done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches c2 rc=$?
python scripts/launch_summary.py gpurun_out/launches_c2_$TAG.csv
