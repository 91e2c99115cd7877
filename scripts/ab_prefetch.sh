for pf in 0 1 0 1; do
  BZK_PREFETCH=$pf python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_pf$pf.json 2>&1
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('pf', sys.argv[2], d['value'], d['kernel_ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_pf$pf.json $pf
done
for pf in 0 1; do
BZK_PREFETCH=$pf ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_round" -c 4 --csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/traffic_pf$pf.csv 2>/dev/null
done
