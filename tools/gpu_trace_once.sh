cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DNCC_TC_TRACE -Ipaper_conf_ipps_moorelk13_b200/csrc -o /tmp/tc_trace tools/microbench/tc_trace.cu -lcuda > gpurun_out/probe_build.log 2>&1
timeout 60 /tmp/tc_trace 32 5 0 > gpurun_out/tc_trace_full.log 2>&1
