mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
B="python bench.py --steps 400 --warmup 10 --no-cpu --no-e2e --no-dp --no-incr --no-dedup --search-budget 0"
show() { python -c "import json,sys; d=json.load(open('$1')); r=d['roofline']; print('%s: %.3f Gcfg/s frac %.3f serial %.1f us' % ('$1', d['value']/1e9, r['frac'], r['kernel_ms_serial']*1e3))" || tail -3 $1.err; }
for k in scan events; do
  ACESO_KERNEL=$k timeout 300 $B > gpurun_out/b_$k.json 2> gpurun_out/b_$k.json.err; show gpurun_out/b_$k.json
  ACESO_KERNEL=$k ACESO_TILES_PER_WARP=1 timeout 300 $B --no-overlap-hint > gpurun_out/b_${k}_nh.json 2> gpurun_out/b_${k}_nh.json.err; show gpurun_out/b_${k}_nh.json
done
for w in gpt-1k; do for k in scan events; do
  ACESO_KERNEL=$k timeout 300 $B --config $w --batch 131072 --steps 40 > gpurun_out/b_${w}_$k.json 2> gpurun_out/b_${w}_$k.json.err; show gpurun_out/b_${w}_$k.json
done; done
