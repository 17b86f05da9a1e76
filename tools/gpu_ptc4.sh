cd "${GRAFT_REPO_ROOT:-/root/repo}"
for n in 3 4 6 8; do echo "nab $n"; NCC_PIV_TC_NAB=$n python tools/piv_tc_prof.py 3 1 2>&1 | tail -30 | tr -d '\n '; echo; NCC_PIV_TC_EXP=8 NCC_PIV_TC_NAB=$n python tools/piv_tc_prof.py 3 1 2>&1 | tail -30 | tr -d '\n '; echo; done > gpurun_out/ptc_nab3.txt 2>&1
