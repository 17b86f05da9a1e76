#!/bin/bash
# Iteration run: build, the named GPU test files, the A/B experiments of tools/gpu_exp.sh.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest -q -x ${TESTS:-tests/test_gpu_tc.py} > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
[ -n "$EXP" ] && bash tools/gpu_exp.sh
rm -rf gpurun_out/jitc
true
