#!/bin/bash
# TM iteration: GPU TM/TC tests, cfg2 + cfg5 bench, ncu of the tensor-core numerator (cfg2).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
timeout 900 python -m pytest tests -q -m gpu -k "tm or tc or roi or ssd" -x > gpurun_out/pytest_tm.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tm.log
timeout 600 python bench.py --workload cfg2 --steps 20 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err
timeout 600 python bench.py --workload cfg5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg5.json 2> gpurun_out/bench_cfg5.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tm_tc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_cfg2.log 2>&1
rm -rf gpurun_out/jitc
