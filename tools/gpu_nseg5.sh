#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for n in 1 2 3 4; do
  NCC_TC_NSEG=$n timeout 300 python bench.py --workload cfg5 --steps 5 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg5_nseg$n.json 2>gpurun_out/b5.err
done
