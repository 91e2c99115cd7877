#!/bin/bash
# round-1 TMA (3 stages) A/B + parity, m0lit passes of 2 vs 3 rounds, c5 strong scaling (1 rank, and 2
# ranks on one GPU over gloo: gather to rank 0 + golden per-proof digests)
TAG=${1:-r02d}
mkdir -p gpurun_out
BZK_TMA=1 timeout 900 python -m pytest tests/test_gpu_fullrange.py tests/test_gpu_parity.py -m gpu -q -x -k "sweep or config or ragged or host or given" > gpurun_out/pytest_tma1_$TAG.log 2>&1; tail -2 gpurun_out/pytest_tma1_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d['roofline'];print(sys.argv[2], d['value'], d.get('scaling'), d['kernel_ms_per_step'], r['bound'], r['frac'], r['kernel'], d['clocks'].get('sm_mhz'), d.get('golden_check'), d.get('proofs_gathered'))" $1 $2 || tail -4 ${1%.json}.err; }
for v in "BZK_MULTI_M=2" "BZK_MULTI_M=3"; do
  env $v timeout 600 python bench.py --config m0lit --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_m0lit_${v}_$TAG.json 2>gpurun_out/bench_m0lit_${v}_$TAG.err
  summ gpurun_out/bench_m0lit_${v}_$TAG.json "m0lit $v"
done
for v in "BZK_TMA=-1" "BZK_TMA=1"; do
  env $v timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c2_${v}_$TAG.json 2>gpurun_out/bench_c2_${v}_$TAG.err
  summ gpurun_out/bench_c2_${v}_$TAG.json "c2 $v"
done
timeout 900 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c5_w1_$TAG.json 2>gpurun_out/bench_c5_w1_$TAG.err
summ gpurun_out/bench_c5_w1_$TAG.json "c5 W=1"
BZK_BENCH_DEVICE=0 BZK_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --config c5 --batch 2048 --wave 512 --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_c5_w2gloo_$TAG.json 2>gpurun_out/bench_c5_w2gloo_$TAG.err
summ gpurun_out/bench_c5_w2gloo_$TAG.json "c5 W=2 gloo one GPU"
