#!/bin/bash
# PIV tensor-core iteration: parity tests, cfg3/cfg4 bench lines, one ncu capture per config.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_piv_tc.py -x -q > gpurun_out/ptc_test.log 2>&1; echo rc=$? >> gpurun_out/ptc_test.log
for w in cfg3 cfg4; do
  timeout 300 python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/ptc_bench_$w.json 2>gpurun_out/ptc_bench_$w.err
done
if [ -n "$NCU" ]; then
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:piv_tc -s 2 -c 2 -o gpurun_out/ptc3 -f python tools/piv_one.py 3 1 > gpurun_out/ptc3_ncu.log 2>&1
  timeout 400 ncu --set full --clock-control none --import-source on -k regex:piv_tc -s 2 -c 2 -o gpurun_out/ptc4 -f python tools/piv_one.py 4 2 > gpurun_out/ptc4_ncu.log 2>&1
fi
python tools/timeline.py 3 > gpurun_out/ptc_tl3.txt 2>&1
