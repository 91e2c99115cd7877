#!/bin/bash
# Round-2 last evidence run (r02fin + Goldilocks sizing fix, unreduced TC deltas, small CUDA-core rounds, d = 3
# on the tensor cores): GPU suite + smoke, every bench line, reference arm, launch lists of c2 and c3,
# ncu --set full of the top kernels, DRAM traffic per kernel kind.  (compute-sanitizer is closed on
# this pool: bounds are covered by the parity suite's ragged / extreme shapes.)
TAG=${1:-r02last}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests/ -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo smoke rc=$?; tail -1 gpurun_out/smoke_$TAG.log
summ() { python -c "import json,sys;d=json.load(open(sys.argv[1]));r=d.get('roofline',{});print(sys.argv[2], d['value'], d.get('unit'), d['ms_per_step'], r.get('bound'), r.get('frac'), r.get('kernel'), d['clocks'].get('sm_mhz'), d['clocks'].get('samples'), d['clocks'].get('reasons'), (d.get('golden_check') or {}).get('mismatches'), (d.get('golden_check') or {}).get('proofs_checked'), d.get('kernel_ms_per_step'))" $1 $2 || tail -4 ${1%.json}.err; }
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_c2_$TAG.json 2> gpurun_out/bench_c2_$TAG.err; summ gpurun_out/bench_c2_$TAG.json c2
for cfg in c3 c5 m0 m0lit g2 mk20 mk20f enc20; do
  timeout 1200 python bench.py --config $cfg --steps 10 --warmup 3 > gpurun_out/bench_${cfg}_$TAG.json 2> gpurun_out/bench_${cfg}_$TAG.err; summ gpurun_out/bench_${cfg}_$TAG.json $cfg
done
timeout 600 python bench.py --config c1 --steps 4000 --warmup 50 > gpurun_out/bench_c1_$TAG.json 2> gpurun_out/bench_c1_$TAG.err; summ gpurun_out/bench_c1_$TAG.json c1
timeout 600 python bench.py --config zk20 --steps 10 --warmup 3 > gpurun_out/bench_zk20_$TAG.json 2> gpurun_out/bench_zk20_$TAG.err; summ gpurun_out/bench_zk20_$TAG.json zk20
for i in 1 2 3; do
  timeout 600 python bench.py --config c4 --steps 5 --warmup 3 > gpurun_out/bench_c4_${i}_$TAG.json 2> gpurun_out/bench_c4_${i}_$TAG.err
  python -c "import json;d=json.load(open('gpurun_out/bench_c4_${i}_$TAG.json'));print('c4 run $i', d['value'], d['overlap'], d['clocks'])"
done
BZK_DIST_FORCE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29513 \
    bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_c2_nccl1_$TAG.json 2> gpurun_out/bench_c2_nccl1_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_c2_nccl1_$TAG.json'));print('nccl1', d['value'], d.get('dist'), {k: v for k, v in d.get('proofs_gathered', {}).items() if k != 'global_digest'}, d.get('golden_check', {}).get('mismatches'))" || tail -5 gpurun_out/bench_c2_nccl1_$TAG.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_c2_$TAG.json 2> gpurun_out/bench_ref_c2_$TAG.err; cat gpurun_out/bench_ref_c2_$TAG.json
for cfg in c2 c3; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${cfg}_$TAG.csv \
      python bench.py --config $cfg --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches $cfg rc=$?
done
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_fused_tc<\(int\)2, \(int\)0, \(bool\)0, \(int\)8" -c 1 -o gpurun_out/prof_k_fused_tc2_c2_$TAG \
    python bench.py --config c2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_f2_$TAG.log 2>&1; echo ncu f2 rc=$?
ncu --set full --clock-control none --import-source on -k regex:k_round1_tc -c 1 -o gpurun_out/prof_k_round1_tc_c2_$TAG \
    python bench.py --config c2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_r1_$TAG.log 2>&1; echo ncu r1 rc=$?
bash scripts/ncu_traffic_r02.sh > /dev/null 2>&1; ls gpurun_out/traffic2_* | wc -l
