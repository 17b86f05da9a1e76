#!/bin/bash
# quick GPU check: all GPU tests, smoke, cfg1/cfg2 bench lines (e2e)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for rep in 1 2 3; do
  timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_q.$rep.json 2>gpurun_out/b2.err
done
timeout 300 python bench.py --workload cfg1 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/sched_cfg1_q.json 2>gpurun_out/b1.err
