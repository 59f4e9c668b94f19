mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
python tools/sanitize_r2.py 2>&1 | tail -7
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t python tools/sanitize_r2.py > gpurun_out/r2_$t.txt 2>&1; echo "$t rc=$?"; tail -3 gpurun_out/r2_$t.txt
done
