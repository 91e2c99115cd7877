#!/bin/bash
# ncu --set full of the final d = 3 kernels (unreduced products on the tensor cores)
TAG=${1:-r02n3}
mkdir -p gpurun_out
for F in 0 1; do
  N=$([ $F = 0 ] && echo 10 || echo 12)
  ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_fused_tc<\(int\)3, \(int\)0, \(bool\)$F" -c 1 -o gpurun_out/prof_k_fused_tc3_${F}_c3_$TAG \
      python bench.py --config c3 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ncu_f3_${F}_$TAG.log 2>&1; echo ncu f3 $F rc=$?
done
