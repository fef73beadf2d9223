#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kfill2 --kernel-name-base demangled -c 4 -o gpurun_out/step2 tools/step_bench2 1 > gpurun_out/step_ncu.log 2>&1
exit 0
