#!/bin/bash
# Full GPU parity suite (-m gpu) on the box; summary in gpurun_out/gpu_tests.log
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout ${T:-2400} python -m pytest tests -m gpu -q ${PYTEST_X:--x} ${PYTEST_K:+-k "$PYTEST_K"} -p no:cacheprovider > gpurun_out/gpu_tests_full.log 2>&1
tail -30 gpurun_out/gpu_tests_full.log | tee gpurun_out/gpu_tests.log
