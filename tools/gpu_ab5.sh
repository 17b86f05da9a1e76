#!/bin/bash
# cfg5 block-combination A/B: default (chained planes), one chain, pure planes, chain lengths.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for v in ${VARS:-"NCC_TC_EXP=0" "NCC_TC_PLANES=0" "NCC_TC_PLANES=1" "NCC_TC_CLEN=4" "NCC_TC_CLEN=16"}; do
  env $v timeout 300 python bench.py --workload cfg5 --no-secondary --no-cpu-baseline --steps 5 > gpurun_out/ab.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('$v', round(d['ms_per_step'],3), round(d['roofline']['kernel_ms'],3), d['correct'], d['config'].get('variant'))" >> gpurun_out/ab5.txt
done
