#!/bin/bash
TAG=${1:-r02r}
mkdir -p gpurun_out
for v in main occ1; do
  if [ $v = main ]; then E=""; else E=BZK_LIB=paper_conf_asplos_lucw0cz25_b200/libbzk_$v.so; fi
  for cfg in c2 c3 m0; do
    env $E timeout 600 python bench.py --config $cfg --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_${v}_$TAG.json 2> gpurun_out/bench_${cfg}_${v}_$TAG.err
    python -c "import json;d=json.load(open('gpurun_out/bench_${cfg}_${v}_$TAG.json'));print('$cfg $v', d['value'], d['kernel_ms_per_step'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/bench_${cfg}_${v}_$TAG.err
  done
done
