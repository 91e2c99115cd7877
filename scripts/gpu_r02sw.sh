#!/bin/bash
# LSB round 1 from 64-byte (a | b) rows (SW64): parity, c2 A/B, launch list
TAG=${1:-r02sw}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_sw_$TAG.log 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/pytest_sw_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in 1 0; do
BZK_R1_SW64=$v timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_sw${v}_$TAG.json 2> gpurun_out/bench_c2_sw${v}_$TAG.err; summ gpurun_out/bench_c2_sw${v}_$TAG.json c2_sw$v
BZK_R1_SW64=$v ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none -k regex:k_round1 --csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/r1_sw${v}_$TAG.csv 2>/dev/null; grep -h "duration\|dram" gpurun_out/r1_sw${v}_$TAG.csv | tail -4 | cut -c1-200
done
