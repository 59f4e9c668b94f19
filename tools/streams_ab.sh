python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
for cfg in gpt3-13b gpt-1k; do for st in 2 3 4; do
  timeout 600 python bench.py --config $cfg --streams $st --no-all --no-e2e --no-cpu --no-dedup --no-dp --search-budget 0 > gpurun_out/st_${cfg}_$st.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/st_${cfg}_$st.json')); print('$cfg', $st, round(d['roofline']['frac'],4), d['config']['l2'])"
done; done
