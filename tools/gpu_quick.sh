#!/bin/bash
# Quick GPU iteration: build, parity suite, default bench (no cpu/e2e legs), optional extra command.
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 | tee gpurun_out/gpu_tests.log
timeout 300 python bench.py --no-cpu --no-e2e --no-dp > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
python -c "import json; d=json.load(open('gpurun_out/bench_quick.json')); r=d['roofline']; print('%.3f Gcfg/s frac %.3f serial %.1f us frac_serial %.3f' % (d['value']/1e9, r['frac'], r['kernel_ms_serial']*1e3, r['frac_serial']))"
[ -n "$1" ] && bash -c "$1"
exit 0
