#!/bin/bash
# quick GPU check: all GPU tests, timelines, cfg1/2/3 bench lines
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python tools/timeline.py 2 5 > gpurun_out/tl2.json 2>/dev/null
NCC_TC_SEPARATE_SPLIT=1 python tools/timeline.py 2 5 > gpurun_out/tl2_sep.json 2>/dev/null
for rep in 1 2; do
  timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_q.$rep.json 2>gpurun_out/b2.err
  NCC_TC_SEPARATE_SPLIT=1 timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_sep.$rep.json 2>gpurun_out/b2.err
done
timeout 300 python bench.py --workload cfg3 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/sched_cfg3_q.json 2>gpurun_out/b3.err
