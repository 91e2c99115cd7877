#!/bin/bash
# Round-2 evidence run with the tensor-core defaults (k_round1_tc, k_fused_tc, k_multi_tc): GPU suite +
# smoke, every bench line, the reference arm, the c2 launch list, ncu --set full of the top kernels,
# DRAM traffic per kernel kind, compute-sanitizer of the round-2 kernels.
TAG=${1:-r02y}
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
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_c2_$TAG.json 2> gpurun_out/bench_ref_c2_$TAG.err; cat gpurun_out/bench_ref_c2_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_$TAG.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches rc=$?
for K in k_fused_tc k_round1_tc; do
  ncu --set full --clock-control none --import-source on -k regex:$K -c 1 -o gpurun_out/prof_${K}_c2_$TAG \
      python bench.py --config c2 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_${K}_$TAG.log 2>&1; echo ncu $K rc=$?
done
ncu --set full --clock-control none --import-source on -k regex:k_multi_tc -c 1 -o gpurun_out/prof_k_multi_tc_m0lit_$TAG \
    python bench.py --config m0lit --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_k_multi_tc_$TAG.log 2>&1; echo ncu multi rc=$?
bash scripts/ncu_traffic_r02.sh > /dev/null 2>&1; ls gpurun_out/traffic2_* | wc -l
bash scripts/sanitize_r02.sh $TAG
