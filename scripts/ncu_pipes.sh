#!/bin/bash
# per-pipe utilisation of the round kernels and the mont_mul micro-benchmark (under gpurun)
TAG=${1:-x}
M=sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fmaheavy.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fmalite.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fmalite.sum,smsp__inst_executed.sum,launch__registers_per_thread
ncu --metrics $M --clock-control none -k regex:"k_round|k_bench" -c 6 --csv python -c "
import sys; sys.path.insert(0,'.')
from paper_conf_asplos_lucw0cz25_b200 import bzk
import torch; torch.cuda.init()
print(bzk.bzk_debug_bench(3, 256)); print(bzk.bzk_debug_bench(0, 256))
" > gpurun_out/pipes_bench_$TAG.csv 2>&1
ncu --metrics $M --clock-control none -k regex:"k_round" -c 2 --csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --batch 256 > gpurun_out/pipes_round_$TAG.csv 2>&1
