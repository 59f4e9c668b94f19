#!/bin/bash
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for split in 1 2; do for st in 1 2 4 8; do
  r=$(ACESO_SPLIT=$split timeout 300 python bench.py --steps 400 --warmup 20 --no-cpu --no-e2e --streams $st 2>&1 | tail -1)
  echo "split=$split streams=$st: $(echo "$r" | python -c "import json,sys; d=json.load(sys.stdin); print('%.3f Gcfg/s  ms/step %.4f kernel %.1f us' % (d['value']/1e9, d['ms_per_step'], d['roofline']['kernel_ms_serial']*1e3))" 2>&1 | tail -1)"
done; done
