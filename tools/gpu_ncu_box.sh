#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:box2d -s 6 -c 1 -o gpurun_out/prof_box -f \
   python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/ncu_box.log 2>&1
ncu -i gpurun_out/prof_box.ncu-rep --page details --csv > gpurun_out/prof_box.details.csv 2>&1
ncu -i gpurun_out/prof_box.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_box.source.csv 2>&1
rm -f gpurun_out/prof_box.ncu-rep
