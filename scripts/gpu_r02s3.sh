#!/bin/bash
# d = 3 round 1 with two TMA stages (8 or 9 compute warps): parity, c3, launch lists
TAG=${1:-r02s3}
mkdir -p gpurun_out
D=$PWD/paper_conf_asplos_lucw0cz25_b200
for lib in main nw9; do
  if [ $lib = main ]; then L=$D/libbzk.so; else L=$D/libbzk_$lib.so; fi
  BZK_LIB=$L timeout 1200 python -m pytest tests/test_gpu_d3_tc.py -x -q > gpurun_out/pytest_${lib}_$TAG.log 2>&1; echo "pytest $lib rc=$?"; tail -1 gpurun_out/pytest_${lib}_$TAG.log
  BZK_LIB=$L ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_${lib}_$TAG.csv \
      python bench.py --config c3 --steps 1 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
  echo $lib; python scripts/launch_summary.py gpurun_out/launches_c3_${lib}_$TAG.csv | grep fused
done
timeout 900 python bench.py --config c3 --steps 10 --warmup 3 > gpurun_out/bench_c3_$TAG.json 2> gpurun_out/bench_c3_$TAG.err
python -c "import json;d=json.load(open('gpurun_out/bench_c3_$TAG.json'));print('c3 main', d['value'], d['kernel_ms_per_step'], d['clocks']['sm_mhz'])"
