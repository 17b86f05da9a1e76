#!/bin/bash
# Round-end evidence on one B200: build, smoke, every GPU test, the default bench line (cfg2 +
# cfg3/4/5 secondaries) and per-config lines, the reference arm, ncu launch lists (cold-cache,
# serialised: shares, not absolutes) and one --set full capture per dominant kernel, summarised
# on the box (the .ncu-rep files would exceed the copy-back limit), CUPTI timelines.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export NCC_CACHE_DIR=$PWD/gpurun_out/jitc
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
if [ -z "$SKIP_TESTS" ]; then
  timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
fi
timeout 1200 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for w in cfg1 cfg3 cfg4 cfg5; do
  timeout 900 python bench.py --workload $w --no-secondary > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for w in cfg2 cfg5; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 60 --csv \
     --log-file gpurun_out/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-secondary > /dev/null 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv \
   --log-file gpurun_out/launches_cfg3.csv python tools/piv_one.py 3 4 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tm_tc_kernel -s 3 -c 1 -o gpurun_out/prof_cfg2 -f \
   python tools/tm_one.py 2 5 > gpurun_out/ncu_cfg2.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:tm_tc_kernel -s 1 -c 1 -o gpurun_out/prof_cfg5 -f \
   python tools/tm_one.py 5 2 > gpurun_out/ncu_cfg5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv3 -f \
   python tools/piv_one.py 3 2 > gpurun_out/ncu_piv3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_tc_kernel -s 1 -c 1 -o gpurun_out/prof_piv4 -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_piv4.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:piv_tc_border -s 1 -c 1 -o gpurun_out/prof_piv4b -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_piv4b.log 2>&1
NCC_PIV_TC=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:piv_ws2 -s 1 -c 1 -o gpurun_out/prof_piv4cc -f \
   python tools/piv_one.py 4 8 > gpurun_out/ncu_piv4cc.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv \
   --log-file gpurun_out/launches_cfg4.csv python tools/piv_one.py 4 8 > /dev/null 2>&1
for r in prof_cfg2 prof_cfg5 prof_piv3 prof_piv4 prof_piv4b prof_piv4cc; do
  if [ -f gpurun_out/$r.ncu-rep ]; then
    python tools/ncu_summary.py full gpurun_out/$r.ncu-rep gpurun_out/$r.json > /dev/null 2>&1
    python tools/ncu_regions.py gpurun_out/$r.ncu-rep 25 > gpurun_out/$r.regions.txt 2>&1
    rm -f gpurun_out/$r.ncu-rep
  fi
done
for w in cfg2 cfg3 cfg4 cfg5; do python tools/ncu_summary.py launches gpurun_out/launches_$w.csv gpurun_out/launches_$w.json > /dev/null 2>&1; done
python tools/timeline.py 2 > gpurun_out/timeline_cfg2.txt 2>&1
python tools/timeline.py 5 3 > gpurun_out/timeline_cfg5.txt 2>&1
python tools/tc_prof.py 2 > gpurun_out/tc_prof2.json 2>&1
python tools/tc_error.py 5 1 > gpurun_out/tc_error5s.jsonl 2>&1
python tools/tc_error.py 2 0 > gpurun_out/tc_error2u.jsonl 2>&1
python tools/piv_tc_prof.py 4 8 > gpurun_out/piv_tc_prof4.json 2>&1
timeout 120 /tmp/umma_probe rates > gpurun_out/umma_rates.log 2>&1 || (nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/umma_probe tools/microbench/umma_probe.cu && timeout 120 /tmp/umma_probe rates > gpurun_out/umma_rates.log 2>&1)
rm -rf gpurun_out/jitc
