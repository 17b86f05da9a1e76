#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
(cd tools/microbench; for e in 0 64; do echo "== exp $e"; timeout 60 ./tc_trace 32 5 $e | grep -v "^q="; done) > gpurun_out/tc_trace.log 2>&1
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tm.py tests/test_gpu_ssd.py -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
for rep in 1 2; do
  timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_q.$rep.json 2>gpurun_out/b2.err
done
timeout 300 python bench.py --workload cfg5 --steps 5 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg5_q.json 2>gpurun_out/b5.err
