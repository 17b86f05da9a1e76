#!/bin/bash
# Tensor-core TM iteration: TC/TM/SSD/multi-process GPU tests, cfg2/cfg5 bench lines, launch lists.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest -q -x tests/test_gpu_tc.py tests/test_gpu_tm.py tests/test_gpu_ssd.py tests/test_gpu_rois.py tests/test_gpu_multiproc.py > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
for w in cfg2 cfg5; do
  timeout 600 python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_cfg2.csv \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_cfg5.csv \
   python tools/tm_one.py 5 2 > /dev/null 2>&1
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
rm -rf gpurun_out/jitc
TL_HOST=1 python tools/timeline.py 2 > gpurun_out/timeline_cfg2_host.txt 2>&1
