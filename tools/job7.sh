mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
B="python bench.py --no-cpu --no-e2e --no-dp --no-dedup --no-all --search-budget 0 --steps 20 --warmup 5"
show() { python -c "import json,sys; d=json.load(open('$1')); r=d['roofline']; print('%s: %.4f Gcfg/s frac %.3f serial %.3f' % ('$1', d['value']/1e9, r['frac'], r['frac_serial']))" || tail -3 $1.err; }
for st in 1 2 4; do $B --streams $st > gpurun_out/k1_s$st.json 2> gpurun_out/k1_s$st.json.err; show gpurun_out/k1_s$st.json; done
ACESO_MINB=2 $B > gpurun_out/k1_m2.json 2> gpurun_out/k1_m2.json.err; show gpurun_out/k1_m2.json
ACESO_KERNEL=scan $B > gpurun_out/k1_scan.json 2> gpurun_out/k1_scan.json.err; show gpurun_out/k1_scan.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -o gpurun_out/r2_ev1k python tools/prof_one.py gpt-1k 131072 2 > gpurun_out/ncu_ev1k.log 2>&1
tail -1 gpurun_out/ncu_ev1k.log
