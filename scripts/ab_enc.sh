for v in main g2 g2t256 g4t256; do
  if [ $v = main ]; then E=""; else E=BZK_LIB=paper_conf_asplos_lucw0cz25_b200/libbzk_$v.so; fi
  env $E python -m pytest tests/test_gpu_encoder.py -x -q 2>&1 | tail -1
  env $E python bench.py --config enc20 --steps 3 --warmup 2 --no-e2e --no-cpu > gpurun_out/ab_enc_$v.json 2>&1
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_enc_$v.json $v || tail -2 gpurun_out/ab_enc_$v.json
done
