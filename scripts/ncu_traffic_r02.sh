#!/bin/bash
# DRAM bytes of every sum-check / encoder launch of one bench step per config (ncu, 3 metrics)
mkdir -p gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
for c in c2 c3 g2 m0 m0lit; do
  ncu --metrics $M --clock-control none -k regex:"k_round|k_gl_round|k_multi|k_fused" --csv \
      python bench.py --config $c --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/traffic2_$c.csv 2>/dev/null
done
ncu --metrics $M --clock-control none -k regex:"k_spmv" --csv \
    python bench.py --config enc20 --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/traffic2_enc20.csv 2>/dev/null
ls -la gpurun_out/traffic2_*
