#!/bin/bash
# event kernel bring-up: build, parity, quick bench of the kernel variants
python __graft_entry__.py > gpurun_out/build_ev.log 2>&1 || { tail -30 gpurun_out/build_ev.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for v in "events 3" "events 2" "quad 3"; do
  set -- $v
  ACESO_KERNEL=$1 ACESO_MINB=$2 timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu --search-budget 0 $BENCH_ARGS 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print('$1 minb $2', round(d['value']/1e9,3), 'Gcfg/s frac', round(r['frac'],3), 'serial ms', round(r.get('kernel_ms_serial'),4), round(r.get('frac_serial'),3))"
done
