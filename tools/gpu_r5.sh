#!/bin/bash
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for w in cfg3 cfg4 cfg2; do
  timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_ncc_kernel -s 2 -c 1 -o gpurun_out/prof_cfg4 -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_cfg4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_ncc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg3 -f \
   python bench.py --workload cfg3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3.log 2>&1
