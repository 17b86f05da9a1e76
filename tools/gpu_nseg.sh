#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for n in 3 4 5 6 7 8; do
  NCC_TC_NSEG=$n timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_nseg$n.json 2>gpurun_out/b2.err
done
