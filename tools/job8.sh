mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
B="python bench.py --no-cpu --no-e2e --no-dp --no-dedup --no-all --search-budget 0 --warmup 5"
show() { python -c "import json,sys; d=json.load(open('$1')); r=d['roofline']; print('%s: %.4f Gcfg/s frac %.3f serial %.3f' % ('$1', d['value']/1e9, r['frac'], r['frac_serial']))" || tail -3 $1.err; }
for w in gpt3-13b t5 wrn gpt3-1.3b; do for m in 2 3; do
  ACESO_MINB=$m $B --config $w --steps 200 > gpurun_out/m_${w}_$m.json 2> gpurun_out/m_${w}_$m.json.err; show gpurun_out/m_${w}_$m.json
done; done
for m in 2 3; do ACESO_MINB=$m $B --config gpt-1k --steps 20 --batch 1048576 > gpurun_out/m_1m_$m.json 2> gpurun_out/m_1m_$m.json.err; show gpurun_out/m_1m_$m.json; done
