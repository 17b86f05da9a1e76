#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for tu in 16 24 32 40 48 64 96; do
  NCC_BOX_TU=$tu python tools/timeline.py 2 5 > gpurun_out/tl2_tu$tu.json 2>/dev/null
  NCC_BOX_TU=$tu python tools/timeline.py 3 5 > gpurun_out/tl3_tu$tu.json 2>/dev/null
done
