mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
timeout 1200 python -m pytest tests/test_gpu_dims.py -q -x -p no:cacheprovider 2>&1 | tail -15
