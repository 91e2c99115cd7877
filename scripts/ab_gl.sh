python -m pytest tests/test_gpu_goldilocks.py -x -q 2>&1 | tail -1
for v in main mf4 mf1 main; do
  if [ $v = main ]; then E=""; else E=BZK_LIB=paper_conf_asplos_lucw0cz25_b200/libbzk_$v.so; fi
  env $E python bench.py --config g2 --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_gl_$v.json 2>&1
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['kernel_ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_gl_$v.json $v || tail -2 gpurun_out/ab_gl_$v.json
done
