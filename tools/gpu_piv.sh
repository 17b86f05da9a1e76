#!/bin/bash
# PIV iteration: GPU PIV tests, cfg3 + cfg4 bench (default and previous variants), ncu of the WS kernels.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
timeout 900 python -m pytest tests -q -m gpu -k "piv or ssd" -x > gpurun_out/pytest_piv.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_piv.log
timeout 600 python bench.py --workload cfg3 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
NCC_FORCE_VARIANT=piv_sk_32x32_m16_rv12_nt416_w4 timeout 600 python bench.py --workload cfg3 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg3_sk.json 2> gpurun_out/bench_cfg3_sk.err
timeout 600 python bench.py --workload cfg4 --steps ${STEPS:-3} --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg4.json 2> gpurun_out/bench_cfg4.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv4 -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_piv4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv3 -f \
   python tools/piv_one.py 3 1 > gpurun_out/ncu_piv3.log 2>&1
rm -rf gpurun_out/jitc
