#!/bin/bash
# d = 2 fused kernel register cap 112 (__maxnreg__) vs 96, lockstep folds at 112: parity, c2, launch lists
TAG=${1:-r02mr}
mkdir -p gpurun_out
D=$PWD/paper_conf_asplos_lucw0cz25_b200
for lib in main f2; do
  if [ $lib = main ]; then L=$D/libbzk.so; else L=$D/libbzk_$lib.so; fi
  BZK_LIB=$L timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_${lib}_$TAG.log 2>&1; echo "pytest $lib rc=$?"; tail -1 gpurun_out/pytest_${lib}_$TAG.log
done
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for lib in main nr96 f2 main2; do
  case $lib in main*) L=$D/libbzk.so;; *) L=$D/libbzk_$lib.so;; esac
  BZK_LIB=$L timeout 900 python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_${lib}_$TAG.json 2> gpurun_out/bench_c2_${lib}_$TAG.err; summ gpurun_out/bench_c2_${lib}_$TAG.json c2_$lib
done
for lib in main nr96 f2; do
  case $lib in main*) L=$D/libbzk.so;; *) L=$D/libbzk_$lib.so;; esac
  BZK_LIB=$L ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_${lib}_$TAG.csv \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
  echo $lib; python scripts/launch_summary.py gpurun_out/launches_c2_${lib}_$TAG.csv | grep fused
done
