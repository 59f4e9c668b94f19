#!/bin/bash
# every BASELINE workload (1 GPU), short runs; one JSON line per config into $1
out=${1:-gpurun_out/profiles/bench_all.jsonl}
mkdir -p $(dirname $out); : > $out
for cfg in toy-a toy-b gpt3-1.3b gpt3-13b t5 wrn gpt-1k; do
  for dist in search dense; do
    b=65536; st=400
    if [ "$cfg" = "gpt-1k" ]; then b=65536; st=20; fi
    if [ "$cfg" = "toy-a" ] || [ "$cfg" = "toy-b" ]; then b=262144; fi
    timeout 900 python bench.py --config $cfg --dist $dist --batch $b --steps $st --warmup 3 \
      --no-e2e --no-cpu --no-dedup --no-dp --no-all --search-budget 0 2>/dev/null | tail -1 >> $out
  done
done
python - "$out" <<'PY'
import json, sys
for line in open(sys.argv[1]):
    try: d = json.loads(line)
    except Exception: continue
    r = d["roofline"]
    print(f'{d["config"]["workload"]:18s} {d["config"]["distribution"]:6s} {d["value"]/1e9:8.3f} Gcfg/s  '
          f'serial {r["kernel_ms_serial"]*1e3:9.1f} us  frac {r["frac"]:.3f} frac_serial {r["frac_serial"]:.3f}')
PY
