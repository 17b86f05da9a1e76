#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tm.py -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
python tools/timeline.py 5 3 > gpurun_out/tl5.json 2>/dev/null
python tools/timeline.py 2 5 > gpurun_out/tl2.json 2>/dev/null
timeout 300 python bench.py --workload cfg5 --steps 5 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg5_q.json 2>gpurun_out/b5.err
timeout 300 python bench.py --workload cfg2 --steps 30 --warmup 5 --no-cpu-baseline --no-secondary > gpurun_out/sched_cfg2_q.json 2>gpurun_out/b2.err
