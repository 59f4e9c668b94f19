# final checks: full GPU suite, smoke(), sanitizers over tests/sanitize_r2.py
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/gpu_tests_full.log 2>&1; tail -1 gpurun_out/gpu_tests_full.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
bash tools/sanitize_job.sh 2>&1 | grep -E "rc=|SUMMARY"
