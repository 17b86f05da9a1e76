#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
NCC_TC_PLANES=0 python tools/timeline.py 2 > gpurun_out/timeline_cfg2_chain.txt 2>&1
TESTS="tests/test_gpu_tc.py tests/test_gpu_tm.py tests/test_gpu_stream.py tests/test_gpu_ssd.py" bash tools/gpu_iter.sh
NCC_TC_PLANES=1 timeout 600 python -m pytest -q -x tests/test_gpu_tc.py -k "cfg5 or bands or ssd" > gpurun_out/pytest_planes5.log 2>&1
for w in cfg2 cfg5; do python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/bench_$w.json 2>gpurun_out/bench_$w.err; done
