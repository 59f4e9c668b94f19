#!/bin/bash
# Regenerates the measurement artifacts of a round on a B200 (run through gpurun):
#   profiles/<tag>_bench.json        the default bench line (N=1)
#   profiles/<tag>_bench_dense.json  the adversarial (dense-random) distribution
#   profiles/<tag>_launches.csv      ncu launch list (gpu__time_duration.sum, serialized)
#   gpurun_out/<tag>_eval.ncu-rep    ncu --set full capture of one eval launch
tag=${1:-r1}
python __graft_entry__.py > gpurun_out/build_$tag.log 2>&1 || { tail -20 gpurun_out/build_$tag.log; exit 1; }
mkdir -p gpurun_out/profiles
timeout 600 python bench.py > gpurun_out/profiles/${tag}_bench.json 2> gpurun_out/bench_$tag.err; tail -c 3000 gpurun_out/profiles/${tag}_bench.json
timeout 300 python bench.py --dist dense --no-cpu > gpurun_out/profiles/${tag}_bench_dense.json 2>> gpurun_out/bench_$tag.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/profiles/${tag}_launches.csv python bench.py --steps 40 --warmup 5 --no-e2e --no-cpu --no-dedup --no-incr --no-dp --search-budget 0 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"event_kernel|eval_kernel" -s 10 -c 1 \
  -o gpurun_out/${tag}_eval python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu --no-dedup --no-incr --no-dp --search-budget 0 > gpurun_out/ncu_$tag.log 2>&1
tail -2 gpurun_out/ncu_$tag.log
