#!/bin/bash
# k_fused_tc bring-up: parity (d = 2 whole proofs), c2 with and without the tensor-core fused rounds
TAG=${1:-r02ft}
mkdir -p gpurun_out
ORDER=0 timeout 120 python scripts/debug_r1.py 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_round1_tc.py -x -q > gpurun_out/pytest_ft_$TAG.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_ft_$TAG.log
for ft in 1 0; do
  BZK_FUSED_TC=$ft timeout 180 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_ft${ft}_$TAG.json 2> gpurun_out/bench_c2_ft${ft}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_c2_ft${ft}_$TAG.json'));print('ft=$ft', d['value'], d['kernel_ms_per_step'], d['golden_check']['mismatches'], d['clocks']['sm_mhz'])" || tail -3 gpurun_out/bench_c2_ft${ft}_$TAG.err
done
