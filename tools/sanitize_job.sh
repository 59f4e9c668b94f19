# compute-sanitizer (memcheck, racecheck, synccheck) over tests/sanitize_r2.py -> gpurun_out/r2_*.txt
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
for t in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 20 python tests/sanitize_r2.py > gpurun_out/r2_$t.txt 2>&1; echo "$t rc=$?"; tail -2 gpurun_out/r2_$t.txt
done
