#!/bin/bash
# TM tensor-core A/B over env knobs on one workload: WL=cfg2|cfg5 VARS="K=V ..."
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for v in ${VARS}; do
  env $v timeout 300 python bench.py --workload ${WL:-cfg2} --no-secondary --no-cpu-baseline --steps ${STEPS:-20} > gpurun_out/ab.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('${WL:-cfg2}', '$v', round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4), d['correct'], d['config'].get('variant'))" >> gpurun_out/ab_tm.txt
done
