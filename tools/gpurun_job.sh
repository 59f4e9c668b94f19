#!/bin/bash
# helper for gpurun iterations: tests, bench, one ncu capture (tag in $1)
tag=${1:-x}
python __graft_entry__.py > gpurun_out/build_$tag.log 2>&1 || { tail -20 gpurun_out/build_$tag.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 300 python bench.py --steps 200 --warmup 20 --no-cpu --no-e2e 2>&1 | tail -1 > gpurun_out/bench_search_$tag.json; cat gpurun_out/bench_search_$tag.json | python -c "import json,sys; d=json.load(sys.stdin); print('search', d['value']/1e9, 'Gcfg/s', d['roofline']['kernel_ms_serial']*1e3, 'us', d['roofline']['frac'])"
timeout 300 python bench.py --steps 200 --warmup 20 --no-cpu --no-e2e --dist dense 2>&1 | tail -1 > gpurun_out/bench_dense_$tag.json; cat gpurun_out/bench_dense_$tag.json | python -c "import json,sys; d=json.load(sys.stdin); print('dense', d['value']/1e9, 'Gcfg/s', d['roofline']['kernel_ms_serial']*1e3, 'us', d['roofline']['frac'])"
if [ -n "$NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval_kernel -s 10 -c 1 -o gpurun_out/prof_$tag python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu > gpurun_out/ncu_$tag.log 2>&1; tail -2 gpurun_out/ncu_$tag.log
fi
