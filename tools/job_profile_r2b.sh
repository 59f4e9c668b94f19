#!/bin/bash
# Round-2 evidence (second session): default bench line, ncu launch list of the headline bench command, full ncu
# capture of one headline launch and of one GPT-3 1.3B 64K launch (event kernel).
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 500 > gpurun_out/r2b_clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/r2b_bench.json 2> gpurun_out/r2b_bench.err; echo "bench rc=$?"
kill $SMI
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2b_launches.csv \
  python bench.py --steps 20 --warmup 5 --no-all --no-e2e --no-cpu --no-dedup --no-dp --search-budget 0 > gpurun_out/r2b_launches.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -o gpurun_out/r2b_ev1k python tools/prof_one.py gpt-1k 131072 2 > gpurun_out/r2b_ev1k.log 2>&1; echo "ncu 1k rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -o gpurun_out/r2b_ev13 python tools/prof_one.py gpt3-1.3b 65536 2 > gpurun_out/r2b_ev13.log 2>&1; echo "ncu 1.3b rc=$?"
timeout 900 python bench.py --batch 1048576 --no-all --no-e2e --no-cpu --no-dedup --no-dp --search-budget 0 --steps 10 --warmup 3 > gpurun_out/r2b_bench_1k_1m.json 2> gpurun_out/r2b_bench_1k_1m.err; echo "1m rc=$?"
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/gpu_tests_full.log 2>&1; tail -1 gpurun_out/gpu_tests_full.log
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2b_reference.json 2> gpurun_out/r2b_reference.err; echo "ref rc=$?"
for r in r2b_ev1k r2b_ev13; do python tools/ncu_summary.py gpurun_out/$r.ncu-rep 40 > gpurun_out/${r}_summary.txt; python tools/ncu_lines.py gpurun_out/$r.ncu-rep 60 > gpurun_out/${r}_lines.txt; done
ncu -i gpurun_out/r2b_ev1k.ncu-rep --page raw --csv --metrics dram__bytes_read.sum,dram__bytes_write.sum > gpurun_out/r2b_traffic_1k.csv 2>&1
ncu -i gpurun_out/r2b_ev13.ncu-rep --page raw --csv --metrics dram__bytes_read.sum,dram__bytes_write.sum > gpurun_out/r2b_traffic_13.csv 2>&1
