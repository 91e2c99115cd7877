#!/bin/bash
# d = 3 fused rounds with 12 compute warps: parity, c3, launch list, ncu of the d = 3 kernels
TAG=${1:-r02d3b}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_d3_tc.py -x -q > gpurun_out/pytest_d3_$TAG.log 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/pytest_d3_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
timeout 900 python bench.py --config c3 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c3_$TAG.json 2> gpurun_out/bench_c3_$TAG.err; summ gpurun_out/bench_c3_$TAG.json c3
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_$TAG.csv \
    python bench.py --config c3 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches c3 rc=$?
python scripts/launch_summary.py gpurun_out/launches_c3_$TAG.csv
for K in "k_fused_tc<3, 0, 0>" "k_fused_tc<3, 0, 1>"; do
  n=$(echo "$K" | tr -d '<>, ')
  ncu --set full --clock-control none --import-source on -k regex:k_fused_tc --kernel-name-base demangled -k "regex:${K}" -c 1 -o gpurun_out/prof_${n}_c3_$TAG \
      python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_${n}_$TAG.log 2>&1; echo ncu $n rc=$?
done
