#!/bin/bash
# variant sweep: register target x split
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for minb in 2 3; do
  ACESO_NVCC_EXTRA="-DACESO_MINB=$minb" python -c "import paper_conf_eurosys_liumlsmybw24_b200 as A; A.build(force=True)" > /dev/null 2>&1
  for split in 1 2; do
    for dist in search dense; do
      r=$(ACESO_SPLIT=$split timeout 300 python bench.py --steps 200 --warmup 20 --no-cpu --no-e2e --dist $dist 2>&1 | tail -1)
      echo "minb=$minb split=$split $dist: $(echo "$r" | python -c "import json,sys; d=json.load(sys.stdin); print('%.3f Gcfg/s  kernel %.1f us  frac %.3f' % (d['value']/1e9, d['roofline']['kernel_ms_serial']*1e3, d['roofline']['frac']))" 2>&1 | tail -1)"
    done
  done
done
