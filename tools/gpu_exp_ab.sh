#!/bin/bash
# tm_tc_kernel issue-loop timing experiments (NCC_TC_EXP bits; results are wrong with them set):
# the cfg2 numerator time per variant.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for v in ${EXPS:-0 512 1024 2048 3584 0}; do
  NCC_TC_EXP=$v timeout 300 python bench.py --workload cfg2 --no-secondary --no-cpu-baseline --steps 30 > gpurun_out/ab.json 2>/dev/null
  python -c "
import json
d=json.loads(open('gpurun_out/ab.json').read().strip().splitlines()[-1])
print('exp $v', round(d['ms_per_step'],4), round(d['roofline']['kernel_ms'],4))" >> gpurun_out/exp_ab.txt
done
