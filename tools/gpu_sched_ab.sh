#!/bin/bash
# A/B of the TM tensor-core launch schedules (NCC_TM_SCHED, NCC_TC_BOX_LATE) on the cfg2 bench line.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for v in ${SCHEDS:-"NCC_TM_SCHED=3" "NCC_TM_SCHED=5" "NCC_TM_SCHED=4" "NCC_TM_SCHED=0" "NCC_TC_BOX_LATE=1" "NCC_TM_SCHED=3"}; do
  env $v timeout 300 python bench.py --workload cfg2 --no-secondary --no-cpu-baseline --steps 40 > gpurun_out/ab.json 2>/dev/null
  python -c "
import json,sys
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('$v', round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4), d['correct'])" >> gpurun_out/sched_ab.txt
done
