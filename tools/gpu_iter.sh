#!/bin/bash
# Iteration run after a tensor-core kernel change: stage tracer, the TC parity tests, cfg2 / cfg5
# bench lines (no CPU baseline / secondaries).  TESTS overrides the test files.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DNCC_TC_TRACE -Ipaper_conf_ipps_moorelk13_b200/csrc \
  -o /tmp/tc_trace tools/microbench/tc_trace.cu -lcuda > gpurun_out/probe_build.log 2>&1
timeout 60 /tmp/tc_trace 32 5 0 > gpurun_out/tc_trace.log 2>&1
for w in ${WORKLOADS:-cfg2 cfg5}; do
  timeout 600 python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/it_bench_$w.json 2> gpurun_out/it_bench_$w.err
done
timeout 1500 python -m pytest ${TESTS:-tests/test_gpu_tc.py tests/test_gpu_tm.py} -q -x -m gpu > gpurun_out/it_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/it_pytest.log
rm -rf gpurun_out/jitc
if [ -n "$AB_EXP" ]; then
  NCC_TC_EXP=$AB_EXP timeout 600 python bench.py --workload cfg2 --no-secondary --no-cpu-baseline > gpurun_out/it_bench_cfg2_ab.json 2> gpurun_out/it_bench_cfg2_ab.err
fi
