#!/bin/bash
# One GPU session: smoke, full gpu tests, bench lines, ncu launch list + full capture.
set -x
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for w in ${BENCH_WORKLOADS:-cfg2 cfg3 cfg5 cfg4}; do
  timeout 900 python bench.py --workload $w --steps ${STEPS:-10} --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_cfg2.csv \
     python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tm_ncc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
     python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_cfg2.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_ncc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg3 -f \
     python bench.py --workload cfg3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3.log 2>&1
fi
ls -la gpurun_out
