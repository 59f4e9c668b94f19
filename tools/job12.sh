mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -k "cta_shapes" -q -p no:cacheprovider > gpurun_out/shape_tests.log 2>&1; tail -3 gpurun_out/shape_tests.log
for sh in 8,2 8,3 6,3 4,4 4,5 4,6; do
  ACESO_EV_SHAPE=$sh timeout 600 python bench.py --no-cpu --no-e2e --no-dp --no-dedup --search-budget 0 --warmup 5 --steps 20 --all-steps 200 > gpurun_out/shape_$sh.json 2> gpurun_out/shape_$sh.err
  python - "$sh" <<'PY'
import json, sys
d = json.load(open(f"gpurun_out/shape_{sys.argv[1]}.json"))
print(sys.argv[1], "gpt-1k", round(d["roofline"]["frac"], 4), *[(k, round(v["roofline"]["frac"], 4)) for k, v in d.get("all_workloads", {}).items()])
PY
done
