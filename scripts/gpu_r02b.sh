#!/bin/bash
# TMA staging A/B: parity with BZK_TMA=1, then c2/c3/m0 bench lines with TMA off/on
TAG=${1:-r02b}
mkdir -p gpurun_out
BZK_TMA=1 timeout 900 python -m pytest tests/test_gpu_fullrange.py tests/test_gpu_parity.py tests/test_gpu_full.py -m gpu -q -x -k "sweep or config or full or larger or given or ragged or host" > gpurun_out/pytest_tma_$TAG.log 2>&1; tail -5 gpurun_out/pytest_tma_$TAG.log
for cfg in c2 c3 m0; do
  for t in 0 1; do
    BZK_TMA=$t timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_${cfg}_tma${t}_$TAG.json 2> gpurun_out/bench_${cfg}_tma${t}_$TAG.err
    python - <<PY
import json
d=json.load(open("gpurun_out/bench_${cfg}_tma${t}_$TAG.json"))
print("${cfg} tma=${t}", d["value"], d["kernel_ms_per_step"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
PY
  done
done
