#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python tools/timeline.py 2 5 > gpurun_out/tl2.json 2>/dev/null
python tools/timeline.py 3 5 > gpurun_out/tl3.json 2>/dev/null
for rep in 1 2; do
  timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_q.$rep.json 2>gpurun_out/b2.err
  timeout 300 python bench.py --workload cfg3 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/sched_cfg3_q.$rep.json 2>gpurun_out/b3.err
done
