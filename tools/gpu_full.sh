#!/bin/bash
# Full validation: smoke, GPU tests, bench lines (all configs), launch list + ncu of the cfg2 numerator.
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for w in cfg2 cfg1 cfg3 cfg4 cfg5; do
  timeout 900 python bench.py --workload $w --steps ${STEPS:-10} --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_cfg2.csv \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tm_tc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_cfg2.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:tm_tc_kernel -s 1 -c 1 -o gpurun_out/prof_cfg5 -f \
   python tools/tm_one.py 5 2 > gpurun_out/ncu_cfg5.log 2>&1
rm -rf gpurun_out/jitc
