#!/bin/bash
# d = 3 on the tensor cores (k_fused_tc<3, ., FIRST>) + out-of-order MMA issue in k_fused_tc: parity,
# c3 A/B (BZK_D3_TC), c2, launch lists of c2 and c3
TAG=${1:-r02d3}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_d3_tc.py tests/test_gpu_round1_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_d3_$TAG.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_d3_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in 1 0; do
  BZK_D3_TC=$v timeout 900 python bench.py --config c3 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c3_d3tc${v}_$TAG.json 2> gpurun_out/bench_c3_d3tc${v}_$TAG.err; summ gpurun_out/bench_c3_d3tc${v}_$TAG.json c3_d3tc$v
done
timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err; summ gpurun_out/bench_c2_$TAG.json c2
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches c2 rc=$?
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_$TAG.csv \
    python bench.py --config c3 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches c3 rc=$?
python scripts/launch_summary.py gpurun_out/launches_c2_$TAG.csv; python scripts/launch_summary.py gpurun_out/launches_c3_$TAG.csv
