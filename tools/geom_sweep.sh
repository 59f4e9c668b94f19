#!/bin/bash
# Launch-geometry sweep of the default bench workload: tiles per warp per launch x streams.
python __graft_entry__.py > /dev/null 2>&1
for tpw in ${TPWS:-1 2 4}; do
  for st in ${STREAMS:-2 4 8}; do
    ACESO_TILES_PER_WARP=$tpw timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu --no-dedup --no-incr --no-dp --search-budget 0 --streams $st 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print('tpw $tpw streams $st', round(d['value']/1e9,3), 'Gcfg/s frac', round(r['frac'],3), 'serial us', round(r['kernel_ms_serial']*1e3,1))"
  done
done
