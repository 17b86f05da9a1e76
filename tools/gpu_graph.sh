#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
python tools/timeline.py 2 5 > gpurun_out/tl2.json 2>/dev/null
for w in cfg1 cfg2 cfg3; do for g in 0 1; do
  if [ $g = 1 ]; then export NCC_NO_GRAPH=1; else unset NCC_NO_GRAPH; fi
  timeout 300 python bench.py --workload $w --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_${w}_nograph$g.json 2>gpurun_out/b_$w.err
done; done
