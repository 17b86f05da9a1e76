cd "${GRAFT_REPO_ROOT:-/root/repo}"
for e in 8 24 56 9 25 57 15 31; do echo "exp $e"; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py 4 8 2>&1 | tail -30 | tr -d '\n '; echo; done > gpurun_out/ptc_prof6.txt 2>&1
