#!/bin/bash
# ncu capture of the eval kernel for a given env (tag in $1)
tag=$1; shift
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"eval_kernel|event_kernel" -s 10 -c 1 -o gpurun_out/prof_$tag python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu "$@" > gpurun_out/ncu_$tag.log 2>&1; tail -1 gpurun_out/ncu_$tag.log
