#!/bin/bash
# A/B of library builds on the quick bench (headline + all workloads): ab.sh name=libpath[:ENV=V,...] ...
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
for spec in "$@"; do
  name=${spec%%=*}; rest=${spec#*=}; lib=${rest%%:*}; envs=""; [[ "$rest" == *:* ]] && envs=${rest#*:}
  (export ACESO_LIB_PATH=$lib; for e in ${envs//,/ }; do export $e; done
   timeout 600 python bench.py --no-cpu --no-e2e --no-dp --no-dedup --search-budget 0 --all-steps ${ALLSTEPS:-200} > gpurun_out/ab_$name.json 2>gpurun_out/ab_$name.err)
  python -c "import json; d=json.load(open('gpurun_out/ab_$name.json')); print('$name', round(d['roofline']['frac'],4), round(d['roofline'].get('frac_serial',0),3), [(k, round(v['roofline']['frac'],3)) for k,v in d['all_workloads'].items()])" || tail -3 gpurun_out/ab_$name.err
done
