#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_piv.py tests/test_gpu_piv_ws.py tests/test_gpu_ssd.py -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
(cd tools/microbench; timeout 60 ./piv_trace 3 1 | head -5; timeout 60 ./piv_trace 4 1 | head -5) > gpurun_out/piv_trace.log 2>&1
for rep in 1 2; do
  timeout 300 python bench.py --workload cfg3 --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/sched_cfg3_q.$rep.json 2>gpurun_out/b3.err
done
timeout 600 python bench.py --workload cfg4 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/sched_cfg4_q.json 2>gpurun_out/b4.err
