for v in main pf1 pf4; do
  if [ $v = main ]; then E=""; else E=BZK_LIB=paper_conf_asplos_lucw0cz25_b200/libbzk_$v.so; fi
  for c in c3 c2; do
    env $E BZK_PREFETCH=1 python bench.py --config $c --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_pfd_${v}_$c.json 2>&1
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['kernel_ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_pfd_${v}_$c.json "$v $c"
  done
done
