cd $GRAFT_REPO_ROOT
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
timeout 900 python -m pytest tests/test_gpu_tm.py tests/test_gpu_piv.py tests/test_gpu_rois.py tests/test_gpu_ssd.py -q -m gpu -x > gpurun_out/pytest_box.log 2>&1; echo rc=$? >> gpurun_out/pytest_box.log
python tools/stage_times.py 2 3 4 > gpurun_out/stages.jsonl 2>&1
NCC_BOX_TWO_PASS=1 python tools/stage_times.py 2 3 4 >> gpurun_out/stages.jsonl 2>&1
rm -rf gpurun_out/jitc
