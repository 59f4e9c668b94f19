for c in gpt3-1.3b gpt3-13b t5 wrn; do for k in events dense quad; do
  ACESO_KERNEL=$k timeout 600 python bench.py --config $c --no-all --no-cpu --no-e2e --no-dp --no-dedup --search-budget 0 --warmup 5 --steps 200 > gpurun_out/k_${c}_$k.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/k_${c}_$k.json')); print('$c', '$k', d['config'].get('schedule'), d['roofline']['frac'])" 2>&1 | tail -1
done; done
