#!/bin/bash
# Short diagnostic run: tm_tc_kernel stage tracer under timing experiments (TRACE_EXPS), and the
# MMA issue-pattern probe (tools/microbench/issue_probe.cu) with PROBE=1.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -DNCC_TC_TRACE -Ipaper_conf_ipps_moorelk13_b200/csrc \
  -o /tmp/tc_trace tools/microbench/tc_trace.cu -lcuda > gpurun_out/probe_build.log 2>&1
for e in ${TRACE_EXPS:-0 34832 100368 65552}; do
  echo "== exp $e" >> gpurun_out/tc_trace.log
  timeout 60 /tmp/tc_trace 32 5 $e 2>&1 | grep -v 'q=' >> gpurun_out/tc_trace.log
done
if [ -n "$PROBE" ]; then
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -Ipaper_conf_ipps_moorelk13_b200/csrc \
    -o /tmp/issue_probe tools/microbench/issue_probe.cu >> gpurun_out/probe_build.log 2>&1
  timeout 120 /tmp/issue_probe > gpurun_out/issue_probe.log 2>&1
fi
