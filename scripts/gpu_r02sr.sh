#!/bin/bash
# 64-thread CTAs for the late CUDA-core rounds (d = 1 BN254, Goldilocks): parity, m0 / g2 A/B, launch lists
TAG=${1:-r02sr}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_small_rounds.py tests/test_gpu_goldilocks.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_sr_$TAG.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_sr_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], r.get('bound'), r.get('frac'), d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
for cfg in m0 g2; do
  for v in 12 0; do
    BZK_SMALL_ROUND_LOG=$v timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_sr${v}_$TAG.json 2> gpurun_out/bench_${cfg}_sr${v}_$TAG.err; summ gpurun_out/bench_${cfg}_sr${v}_$TAG.json ${cfg}_sr$v
    BZK_SMALL_ROUND_LOG=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${cfg}_sr${v}_$TAG.csv \
        python bench.py --config $cfg --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
    python scripts/launch_summary.py gpurun_out/launches_${cfg}_sr${v}_$TAG.csv | grep -v "generate\|init_consts"
  done
done
