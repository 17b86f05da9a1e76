cd "${GRAFT_REPO_ROOT:-/root/repo}"
for e in 0 1 2 4 8 6 14 7; do echo "exp $e"; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py 4 8 2>&1 | python3 -c "
import json,sys; t=sys.stdin.read(); d=json.loads(t[t.index('{'):]); print({k:(v if not isinstance(v,dict) else {kk:vv for kk,vv in v.items()}) for k,v in d.items() if k in ('mma','producers','epilogue','prep')})"; done > gpurun_out/ptc_exp4.txt 2>&1
for e in 0 2 4 6; do echo "exp $e"; NCC_PIV_TC_EXP=$e python tools/piv_tc_prof.py 3 1 2>&1 | tail -30 | tr -d '\n'; echo; done > gpurun_out/ptc_exp3.txt 2>&1
