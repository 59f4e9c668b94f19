# the default bench line with NVML clocks -> gpurun_out/r2_bench.json, r2_clocks.csv
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 500 > gpurun_out/r2_clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/r2_bench.json 2> gpurun_out/r2_bench.err; echo "bench rc=$?"
kill $SMI
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2_reference.json 2> gpurun_out/r2_reference.err; echo "ref rc=$?"; cat gpurun_out/r2_reference.json
