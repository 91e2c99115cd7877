#!/bin/bash
# usage (under gpurun): bash scripts/gpu_round2.sh <tag> — tests, every bench config, launch list, ncu full
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/ -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
for c in c3 g2 m0 m0lit c4 c1 mk20 mk20f; do
  python bench.py --config $c --steps 3 --warmup 3 --no-e2e > gpurun_out/bench_${c}_$TAG.json 2> gpurun_out/bench_${c}_$TAG.err
  cat gpurun_out/bench_${c}_$TAG.json; tail -2 gpurun_out/bench_${c}_$TAG.err
done
BZK_BENCH_DEVICE=0 BZK_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
   --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 2 --warmup 3 --batch 128 --no-e2e \
   > gpurun_out/bench_2rank_smoke_$TAG.json 2> gpurun_out/bench_2rank_smoke_$TAG.err; cat gpurun_out/bench_2rank_smoke_$TAG.json
python bench.py --impl reference --steps 1 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2>&1; cat gpurun_out/bench_ref_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch_bench_$TAG.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_round -s 0 -c 2 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/ncu_full_$TAG.log 2>&1
bash scripts/ncu_pipes.sh $TAG
ls gpurun_out | wc -l
