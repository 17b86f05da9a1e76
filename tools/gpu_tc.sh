cd $GRAFT_REPO_ROOT; bash tools/gpu_tm.sh
