#!/bin/bash
# Round-2 GPU iteration: parity suite (default = scan kernel), then bench lines of the scan
# kernel and of the round-1 event kernel (same batches), multi-stream and single-stream.
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 1200 python -m pytest tests -m gpu -q -x ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -25 | tee gpurun_out/gpu_tests.log
for k in scan events; do
  for st in 8 1; do
    ACESO_KERNEL=$k timeout 300 python bench.py --steps 200 --warmup 10 --streams $st --no-cpu --no-e2e --no-dp --no-incr --no-dedup --search-budget 0 > gpurun_out/b_${k}_${st}.json 2> gpurun_out/b_${k}_${st}.err
    python -c "import json,sys; d=json.load(open('gpurun_out/b_${k}_${st}.json')); r=d['roofline']; print('$k streams=$st: %.3f Gcfg/s frac %.3f serial %.1f us frac_serial %.3f' % (d['value']/1e9, r['frac'], r['kernel_ms_serial']*1e3, r['frac_serial']))" || tail -5 gpurun_out/b_${k}_${st}.err
  done
done
[ -n "$EXTRA" ] && bash -c "$EXTRA"
exit 0
