#!/bin/bash
# ncu --set full of one event-kernel launch per library build: ncu_ab.sh workload n name=lib ...
mkdir -p gpurun_out
python -c "import oracle, aceso_inputs; oracle.build(); aceso_inputs.build()"
w=$1; n=$2; shift 2
for spec in "$@"; do
  name=${spec%%=*}; lib=${spec#*=}
  ACESO_LIB_PATH=$lib timeout 900 ncu --set full --clock-control none --import-source on -k regex:event_kernel -s 1 -c 1 -f -o gpurun_out/ab_$name python tools/prof_one.py $w $n 2 > gpurun_out/ab_ncu_$name.log 2>&1; echo "ncu $name rc=$?"
done
