for pf in 1 0; do
  for c in c2 m0 c3; do
    BZK_PREFETCH=$pf python bench.py --config $c --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_pf1_${pf}_$c.json 2>&1
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['kernel_ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_pf1_${pf}_$c.json "pf=$pf $c"
  done
done
BZK_PREFETCH=1 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_round" -c 4 --csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu 2>/dev/null | grep dram__bytes_read | awk -F'","' '{print $5, $NF}'
