#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
NCC_TM_SCHED=5 timeout 600 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tm.py tests/test_gpu_ssd.py -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
for s in 3 5; do NCC_TM_SCHED=$s python tools/timeline.py 2 5 > gpurun_out/tl2_$s.json 2>/dev/null; done
for rep in 1 2; do for s in 3 5; do
  NCC_TM_SCHED=$s timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_$s.$rep.json 2>gpurun_out/b2.err
done; done
