#!/bin/bash
# usage (under gpurun): bash scripts/knob_sweep.sh "ENV1=a ENV2=b" "ENV1=c" ...
for cfg in "$@"; do
  echo "== $cfg"
  env $cfg python bench.py --no-e2e --no-cpu --steps 3 --warmup 2 ${BENCH_ARGS} | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['kernel_ms_per_step'], d['roofline']['frac'])"
done
