#!/bin/bash
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/sweep.py tm 2 > gpurun_out/sweep_tm2.jsonl 2> gpurun_out/sweep_tm2.err
timeout 600 python tools/sweep.py tm 5 > gpurun_out/sweep_tm5.jsonl 2> gpurun_out/sweep_tm5.err
for w in cfg2 cfg5; do
  timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tm_ncc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_cfg2.log 2>&1
