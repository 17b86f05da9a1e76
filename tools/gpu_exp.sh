#!/bin/bash
# A/B timing experiments of the tensor-core TM path (env knobs), cfg2 and cfg5 device timings.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
run() {  # name, workload, env...
  local name=$1 w=$2; shift 2
  env "$@" timeout 300 python bench.py --workload $w --no-secondary --no-cpu-baseline --steps 20 > gpurun_out/exp_${name}.json 2> gpurun_out/exp_${name}.err
}
run def2 cfg2
run nowait2 cfg2 NCC_TC_EXP=1
run nodrain2 cfg2 NCC_TC_EXP=2
run fence2 cfg2 NCC_TC_EXP=4
run prefonly2 cfg2 NCC_TC_EXP=16
run def5 cfg5
run nodrain5 cfg5 NCC_TC_EXP=2
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
for f in gpurun_out/exp_*.json; do python -c "
import json,sys; d=json.load(open('$f')); r=d['roofline']; print('$f', d['config']['variant'], round(d['ms_per_step'],4), round(r['kernel_ms'],4), d['correct'], d['clocks']['sm_mhz'])"; done > gpurun_out/exp_summary.txt 2>&1
