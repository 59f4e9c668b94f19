# stream-count sweep of the short-model workloads (bench.py --streams)
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
for cfg in gpt3-1.3b wrn t5; do for st in 4 8 12 16; do
  timeout 600 python bench.py --config $cfg --streams $st --steps 200 --no-all --no-e2e --no-cpu --no-dedup --no-dp --search-budget 0 > gpurun_out/ss_${cfg}_$st.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ss_${cfg}_$st.json')); print('$cfg', $st, round(d['roofline']['frac'],4))"
done; done
