# full GPU suite, then a short headline bench
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/gpu_tests_full.log 2>&1; tail -1 gpurun_out/gpu_tests_full.log
timeout 600 python bench.py --no-cpu --no-e2e --no-dp --no-dedup --search-budget 0 --all-steps 200 > gpurun_out/quick.json 2>/dev/null
python -c "import json; d=json.load(open('gpurun_out/quick.json')); print('headline', d['roofline']['frac'], [(k, round(v['roofline']['frac'],3)) for k,v in d['all_workloads'].items()])"
