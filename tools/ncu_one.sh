#!/bin/bash
# ncu --set full of one eval launch of the default bench (tag = $1), summaries into gpurun_out/
tag=${1:-x}; shift
mkdir -p gpurun_out
[ -f paper_conf_eurosys_liumlsmybw24_b200/libaceso.so ] && [ -z "$NCU_REBUILD" ] || python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"event_kernel|eval_kernel|dense_kernel" -s 10 -c 1 \
  -o gpurun_out/${tag} python bench.py --steps 20 --warmup 5 --streams 1 --no-e2e --no-cpu "$@" > gpurun_out/ncu_$tag.log 2>&1
tail -2 gpurun_out/ncu_$tag.log
python tools/ncu_summary.py gpurun_out/${tag}.ncu-rep > gpurun_out/${tag}_summary.txt 2>&1
python tools/ncu_lines.py gpurun_out/${tag}.ncu-rep 60 > gpurun_out/${tag}_lines.txt 2>&1
cat gpurun_out/${tag}_summary.txt
