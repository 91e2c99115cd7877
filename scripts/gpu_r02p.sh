#!/bin/bash
TAG=${1:-r02p}
mkdir -p gpurun_out
BZK_DUAL=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api.py tests/test_gpu_fullrange.py tests/test_gpu_full.py -m gpu -q -x -k "not cluster and not per_round" > gpurun_out/pytest_dual_$TAG.log 2>&1; tail -2 gpurun_out/pytest_dual_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['clocks'].get('sm_mhz'), d['clocks'].get('samples'), (d.get('golden_check') or {}).get('mismatches'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in 0 1; do
 for cfg in c2 c3 m0; do
  BZK_DUAL=$v timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_dual${v}_$TAG.json 2> gpurun_out/bench_${cfg}_dual${v}_$TAG.err; summ gpurun_out/bench_${cfg}_dual${v}_$TAG.json "$cfg dual=$v"
 done
done
