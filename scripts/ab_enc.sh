for v in k2u1 k2u1t128 k2u2t128 k1u2t128 k2u4t128 k2u1t64; do
  BZK_LIB=paper_conf_asplos_lucw0cz25_b200/libbzk_$v.so python bench.py --config enc20 --steps 3 --warmup 2 --no-e2e --no-cpu > gpurun_out/ab_enc_$v.json 2>&1
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['value'], d['ms_per_step'], d['roofline']['frac'])" gpurun_out/ab_enc_$v.json $v || tail -2 gpurun_out/ab_enc_$v.json
done
