cd $GRAFT_REPO_ROOT
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
for e in 0 4; do timeout 60 tools/microbench/tc_trace 32 4 $e; done > gpurun_out/tc_trace.log 2>&1
timeout 300 python -m pytest tests/test_gpu_tc.py -q -m gpu -x > gpurun_out/pytest_tc.log 2>&1; echo rc=$? >> gpurun_out/pytest_tc.log
if grep -q "rc=0" gpurun_out/pytest_tc.log; then
  NCC_TC=1 python tools/stage_times.py 2 5 > gpurun_out/stages_tc.jsonl 2>&1
else
  NCC_TC=1 CUDA_LAUNCH_BLOCKING=1 timeout 120 compute-sanitizer python -m pytest tests/test_gpu_tc.py -q -m gpu -x -k "64-64-16" > gpurun_out/tc_sanitizer.log 2>&1
fi
rm -rf gpurun_out/jitc
