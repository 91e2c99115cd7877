#!/bin/bash
# k_multi v2 (288-bit REDC, lazy column sums, MSB TMA) parity + m0lit A/B (TMA off/on)
TAG=${1:-r02f}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multiround.py tests/test_gpu_parity.py -m gpu -q -x -k "multiround or given or m0lit" > gpurun_out/pytest_multi_$TAG.log 2>&1; tail -2 gpurun_out/pytest_multi_$TAG.log
BZK_TMA=0 timeout 900 python -m pytest tests/test_gpu_multiround.py -m gpu -q -x > gpurun_out/pytest_multi_notma_$TAG.log 2>&1; tail -2 gpurun_out/pytest_multi_notma_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d['roofline'];print(sys.argv[2], d['value'], d['kernel_ms_per_step'], r['bound'], r['frac'], r.get('imad_frac'), r.get('hbm_frac'), d['clocks'].get('sm_mhz'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in "BZK_TMA=0" "BZK_NOTHING=1"; do
  env $v timeout 600 python bench.py --config m0lit --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_${v}_$TAG.json 2>gpurun_out/bench_m0lit_${v}_$TAG.err
  summ gpurun_out/bench_m0lit_${v}_$TAG.json "m0lit $v"
done
ncu --set full --clock-control none --import-source on -k regex:k_multi -s 0 -c 1 -o gpurun_out/prof_m0lit_$TAG python bench.py --config m0lit --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_m0lit_$TAG.log 2>&1; tail -1 gpurun_out/ncu_m0lit_$TAG.log
