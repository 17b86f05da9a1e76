#!/bin/bash
# quick GPU check: all GPU tests, smoke, cfg1/cfg2 bench lines
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for rep in 1 2; do
  timeout 300 python bench.py --workload cfg1 --steps 30 --warmup 5 > gpurun_out/sched_cfg1_q.$rep.json 2>gpurun_out/b1.err
done
NCC_NO_TINY=1 timeout 300 python bench.py --workload cfg1 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/sched_cfg1_notiny.json 2>>gpurun_out/b1.err
