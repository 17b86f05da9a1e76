cd "${GRAFT_REPO_ROOT:-/root/repo}"
for e in ${EXPS:-0 8}; do echo "exp $e"; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py ${CFG:-4} ${PAIRS:-8} 2>&1 | grep -v "^ok" | tr -d '\n '; echo; done > gpurun_out/ptc_prof7.txt 2>&1
