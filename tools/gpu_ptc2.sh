cd "${GRAFT_REPO_ROOT:-/root/repo}"
timeout 600 python -m pytest tests/test_gpu_piv_tc.py -x -q > gpurun_out/ptc_test.log 2>&1; echo rc=$? >> gpurun_out/ptc_test.log
python tools/piv_tc_prof.py 3 1 > gpurun_out/ptc_prof3.json 2>&1
python tools/piv_tc_prof.py 4 8 > gpurun_out/ptc_prof4.json 2>&1
for w in cfg3 cfg4; do timeout 300 python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/ptc_bench_$w.json 2>gpurun_out/ptc_bench_$w.err; done
