mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -k "two_tiles or gpt_1k" -q -p no:cacheprovider > gpurun_out/sc_tests.log 2>&1; tail -1 gpurun_out/sc_tests.log
for r in 1 2 3; do
  timeout 600 python bench.py --no-cpu --no-e2e --no-dp --no-dedup --no-all --search-budget 0 --warmup 5 --steps 20 > gpurun_out/hl_$r.json 2> gpurun_out/hl_$r.err
  python -c "import json; d=json.load(open('gpurun_out/hl_$r.json')); print($r, d['roofline']['frac'], d['roofline']['frac_serial'])"
done
