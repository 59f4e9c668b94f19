mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -k "two_tiles or gpt_1k or bench_config" -q -p no:cacheprovider > gpurun_out/sc_tests.log 2>&1; tail -3 gpurun_out/sc_tests.log
for sl in 8 4 8 4; do
  ACESO_EV_SLOT=$sl timeout 600 python bench.py --no-cpu --no-e2e --no-dp --no-dedup --search-budget 0 --warmup 5 --steps 20 --all-steps 200 > gpurun_out/slot_$sl.json 2> gpurun_out/slot_$sl.err
  python - "$sl" <<'PY'
import json, sys
d = json.load(open(f"gpurun_out/slot_{sys.argv[1]}.json"))
print(sys.argv[1], "gpt-1k", round(d["roofline"]["frac"], 4), round(d["roofline"]["frac_serial"], 4), *[(k, round(v["roofline"]["frac"], 4)) for k, v in d.get("all_workloads", {}).items()])
PY
done
