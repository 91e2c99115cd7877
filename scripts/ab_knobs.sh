for kv in "BZK_PPT_MAX=128" "BZK_PPT_MAX=256" "BZK_PPT_MAX=1024" "BZK_PPT_MAX=64"; do
  for c in c2 c3 m0; do
    env $kv python bench.py --config $c --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_knob.json 2>&1
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['kernel_ms_per_step'])" gpurun_out/ab_knob.json "$kv $c"
  done
done
