cd "${GRAFT_REPO_ROOT:-/root/repo}"
timeout 600 python -m pytest tests/test_gpu_piv_tc.py -x -q > gpurun_out/ptc_test.log 2>&1; echo rc=$? >> gpurun_out/ptc_test.log
for e in 0 8; do echo "exp $e"; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py 4 8 2>&1 | tail -30 | tr -d '\n '; echo; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py 3 1 2>&1 | tail -30 | tr -d '\n '; echo; done > gpurun_out/ptc_prof5.txt 2>&1
for w in cfg3 cfg4; do timeout 300 python bench.py --workload $w --no-secondary --no-cpu-baseline > gpurun_out/ptc_bench_$w.json 2>gpurun_out/ptc_bench_$w.err; done
