cd $GRAFT_REPO_ROOT
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
echo "== band cfg1"; timeout 300 python -m pytest tests/test_gpu_tm.py -q -m gpu -k cfg1 2>&1 | tail -2
run() { echo "== $*"; CUDA_LAUNCH_BLOCKING=1 timeout 60 python tools/roi_debug2.py "$@" 2>&1 | tail -1 | cut -c1-200; }
run 200 180 16 16 1 1 40 56 0 0
run 200 180 16 16 1 1 40 56 0 4
run 200 180 16 16 1 1 40 56 0 78
run 200 180 16 16 1 1 40 56 16 0
run 200 180 16 16 1 1 40 56 40 0
run 200 180 16 16 1 1 8 64 40 0
run 200 180 16 16 1 1 8 64 0 0
run 200 180 16 16 2 1 8 64 0 0 0 0
run 200 180 16 16 1 2 8 64 0 0 0 0
run 200 176 16 16 1 1 40 56 0 0
run 256 256 16 16 1 1 40 56 0 0
