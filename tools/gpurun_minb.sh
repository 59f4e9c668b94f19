#!/bin/bash
# register-target sweep (ACESO_MINB) in serial and concurrent bench modes
for minb in 2 3 4; do
  ACESO_NVCC_EXTRA="-DACESO_MINB=$minb" python -c "import paper_conf_eurosys_liumlsmybw24_b200 as A; A.build(force=True)" > /dev/null 2>&1
  for st in 1 4 8; do
    r=$(ACESO_SPLIT=1 timeout 300 python bench.py --steps 400 --warmup 20 --no-cpu --no-e2e --search-budget 0 --streams $st 2>&1 | tail -1)
    echo "minb=$minb streams=$st: $(echo "$r" | python -c "import json,sys; d=json.load(sys.stdin); print('%.3f Gcfg/s serial %.1f us' % (d['value']/1e9, d['roofline']['kernel_ms_serial']*1e3))" 2>&1 | tail -1)"
  done
done
