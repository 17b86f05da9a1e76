#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
NCC_TM_SCHED=4 python tools/timeline.py 2 > gpurun_out/timeline_cfg2_s4.txt 2>&1
TL_HOST=1 TL_BATCH=8 python tools/timeline.py 2 2 > gpurun_out/timeline_cfg2_host8.txt 2>&1
python tools/paper_sweeps.py 6.16 > gpurun_out/sweep616.jsonl 2> gpurun_out/sweep616.err
NCC_TM_SCHED=4 TESTS="tests/test_gpu_tc.py tests/test_gpu_stream.py" bash tools/gpu_iter.sh
TESTS="tests/test_gpu_piv.py tests/test_jit.py" bash tools/gpu_iter.sh; cp gpurun_out/pytest_iter.log gpurun_out/pytest_piv.log
rm -rf gpurun_out/jitc
