#!/bin/bash
# d = 2 fused rounds with 6 compute warps (3 CTAs per SM) vs 8 (2 per SM): parity of the variant, c2 A/B,
# launch lists
TAG=${1:-r02nw}
mkdir -p gpurun_out
V=$PWD/paper_conf_asplos_lucw0cz25_b200/libbzk_nw6.so
timeout 1800 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
BZK_LIB=$V timeout 1500 python -m pytest tests/test_gpu_round1_tc.py tests/test_gpu_full.py -x -q > gpurun_out/pytest_nw6_$TAG.log 2>&1; echo "pytest nw6 rc=$?"
tail -2 gpurun_out/pytest_nw6_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for lib in nw6 main nw6b mainb; do
  case $lib in nw6*) L=$V;; *) L=$PWD/paper_conf_asplos_lucw0cz25_b200/libbzk.so;; esac
  BZK_LIB=$L timeout 900 python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_${lib}_$TAG.json 2> gpurun_out/bench_c2_${lib}_$TAG.err; summ gpurun_out/bench_c2_${lib}_$TAG.json c2_$lib
done
for lib in main nw6; do
  case $lib in nw6*) L=$V;; *) L=$PWD/paper_conf_asplos_lucw0cz25_b200/libbzk.so;; esac
  BZK_LIB=$L ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_${lib}_$TAG.csv \
      python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
  python scripts/launch_summary.py gpurun_out/launches_c2_${lib}_$TAG.csv | grep -v generate
done
