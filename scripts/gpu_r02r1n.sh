#!/bin/bash
# k_round1_tc without D-prep warps (block sums aa, ab, ba, bb straight from the TMA tiles): parity,
# c2, launch list, ncu of the new round-1 kernel and of the d = 3 fused kernel
TAG=${1:-r02r1n}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_r1n_$TAG.log 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/pytest_r1n_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err; summ gpurun_out/bench_c2_$TAG.json c2
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches c2 rc=$?
python scripts/launch_summary.py gpurun_out/launches_c2_$TAG.csv
ncu --set full --clock-control none --import-source on -k regex:k_round1_tc -c 1 -o gpurun_out/prof_k_round1_tc_c2_$TAG \
    python bench.py --config c2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_r1_$TAG.log 2>&1; echo ncu r1 rc=$?
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_fused_tc<3, 0, 0>" -c 1 -o gpurun_out/prof_k_fused_tc3_c3_$TAG \
    python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_f3_$TAG.log 2>&1; echo ncu f3 rc=$?
