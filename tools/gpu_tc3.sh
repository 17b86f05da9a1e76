#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
NCC_TC_BOX_LATE=0 python tools/timeline.py 2 > gpurun_out/timeline_cfg2_early.txt 2>&1
TESTS="tests/test_gpu_tc.py tests/test_gpu_tm.py tests/test_gpu_stream.py tests/test_gpu_ssd.py tests/test_gpu_rois.py" bash tools/gpu_iter.sh
NCC_NO_GRAPH=1 timeout 600 python -m pytest -q -x tests/test_gpu_tc.py -k "cfg2 or host or bands" > gpurun_out/pytest_nograph.log 2>&1
python bench.py --workload cfg2 --no-secondary --no-cpu-baseline > gpurun_out/bench_cfg2.json 2>gpurun_out/bench_cfg2.err
