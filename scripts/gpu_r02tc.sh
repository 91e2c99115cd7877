#!/bin/bash
# k_multi_tc bring-up: parity of the known-challenge passes, smoke, m0lit with and without the tensor cores
TAG=${1:-r02tc}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multiround.py -x -q > gpurun_out/pytest_multi_$TAG.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_multi_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
for tc in 1 0; do
  BZK_MULTI_TC=$tc timeout 600 python bench.py --config m0lit --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_tc${tc}_$TAG.json 2> gpurun_out/bench_m0lit_tc${tc}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_m0lit_tc${tc}_$TAG.json'));print('tc=$tc', d['value'], d['kernel_ms_per_step'], d['roofline']['kernel'], d['roofline']['bound'], d['roofline']['frac'], d['clocks']['sm_mhz'])" || tail -5 gpurun_out/bench_m0lit_tc${tc}_$TAG.err
done
