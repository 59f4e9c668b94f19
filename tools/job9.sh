mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
python tools/prof_one.py gpt3-1.3b 8192 2 --check 2>&1 | grep mismatches
python tools/prof_one.py t5 4096 2 --check 2>&1 | grep mismatches
python tools/prof_one.py gpt-1k 1024 2 --check 2>&1 | grep mismatches
B="python bench.py --no-cpu --no-e2e --no-dp --no-dedup --no-all --search-budget 0 --warmup 5"
show() { python -c "import json,sys; d=json.load(open('$1')); r=d['roofline']; print('%s: %.4f Gcfg/s frac %.3f serial %.3f' % ('$1', d['value']/1e9, r['frac'], r['frac_serial']))" || tail -3 $1.err; }
for w in gpt-1k gpt3-1.3b gpt3-13b t5 wrn; do
  st=200; [ $w = gpt-1k ] && st=20
  $B --config $w --steps $st > gpurun_out/n_$w.json 2> gpurun_out/n_$w.json.err; show gpurun_out/n_$w.json
  ACESO_LIB_PATH=$PWD/paper_conf_eurosys_liumlsmybw24_b200/libaceso_legacy_rc.so $B --config $w --steps $st > gpurun_out/o_$w.json 2> gpurun_out/o_$w.json.err; show gpurun_out/o_$w.json
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -o gpurun_out/r2_ev1k_rcq python tools/prof_one.py gpt-1k 131072 2 > gpurun_out/ncu.log 2>&1; tail -1 gpurun_out/ncu.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -o gpurun_out/r2_ev13_rcq python tools/prof_one.py gpt3-1.3b 65536 2 > gpurun_out/ncu2.log 2>&1; tail -1 gpurun_out/ncu2.log
