#!/bin/bash
# fold2 (two folds of a pair group in lockstep) A/B: parity with the variant library, c2 and c3 with
# both, launch lists
TAG=${1:-r02f2}
mkdir -p gpurun_out
V=paper_conf_asplos_lucw0cz25_b200/libbzk_fold2.so
BZK_LIB=$PWD/$V timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_d3_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_f2_$TAG.log 2>&1; echo "pytest fold2 rc=$?"
tail -2 gpurun_out/pytest_f2_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for lib in main fold2; do
  if [ $lib = main ]; then L=$PWD/paper_conf_asplos_lucw0cz25_b200/libbzk.so; else L=$PWD/$V; fi
  for cfg in c2 c3; do
    BZK_LIB=$L timeout 900 python bench.py --config $cfg --steps 6 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_${lib}_$TAG.json 2> gpurun_out/bench_${cfg}_${lib}_$TAG.err; summ gpurun_out/bench_${cfg}_${lib}_$TAG.json ${cfg}_$lib
    BZK_LIB=$L ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${cfg}_${lib}_$TAG.csv \
      python bench.py --config $cfg --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
    python scripts/launch_summary.py gpurun_out/launches_${cfg}_${lib}_$TAG.csv | grep -v generate
  done
done
