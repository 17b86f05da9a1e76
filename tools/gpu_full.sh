#!/bin/bash
# Full validation: smoke, GPU tests, bench lines (all configs), launch list + ncu of the numerators.
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for w in cfg2 cfg1 cfg3 cfg4 cfg5; do
  timeout 900 python bench.py --workload $w --steps ${STEPS:-10} --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_cfg2.csv \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tm_tc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_cfg2.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:tm_tc_kernel -s 1 -c 1 -o gpurun_out/prof_cfg5 -f \
   python tools/tm_one.py 5 2 > gpurun_out/ncu_cfg5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv4 -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_piv4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv3 -f \
   python tools/piv_one.py 3 1 > gpurun_out/ncu_piv3.log 2>&1
# summarise on the box (the .ncu-rep files would exceed the 64 MiB copy-back limit)
for r in prof_cfg2 prof_cfg5 prof_piv4 prof_piv3; do
  if [ -f gpurun_out/$r.ncu-rep ]; then
    python tools/ncu_summary.py full gpurun_out/$r.ncu-rep gpurun_out/$r.json > /dev/null 2>&1
    python tools/ncu_regions.py gpurun_out/$r.ncu-rep 25 > gpurun_out/$r.regions.txt 2>&1
    rm -f gpurun_out/$r.ncu-rep
  fi
done
python tools/ncu_summary.py launches gpurun_out/launches_cfg2.csv gpurun_out/launches_cfg2.json > /dev/null 2>&1
rm -rf gpurun_out/jitc
if [ -x tools/microbench/tc_trace ]; then
  for e in 0 65552 34832; do echo "== exp $e"; timeout 60 tools/microbench/tc_trace 32 5 $e; done > gpurun_out/tc_trace.log 2>&1
fi
python tools/stage_times.py 2 3 4 > gpurun_out/stages.jsonl 2>&1
