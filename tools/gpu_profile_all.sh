#!/bin/bash
# Round artifacts: tools/profile_round.sh (bench line, dense line, ncu launch list, ncu full
# capture) + every workload (tools/bench_all.sh) + ncu summaries; all under gpurun_out/.
tag=${1:-r1}
bash tools/profile_round.sh $tag
python tools/ncu_summary.py gpurun_out/${tag}_eval.ncu-rep 30 > gpurun_out/profiles/${tag}_eval_summary.txt 2>&1
python tools/ncu_lines.py gpurun_out/${tag}_eval.ncu-rep 60 > gpurun_out/profiles/${tag}_eval_lines.txt 2>&1
bash tools/bench_all.sh gpurun_out/profiles/${tag}_bench_all.jsonl
