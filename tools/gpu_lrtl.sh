#!/bin/bash
# C3 timeline session (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 300 python tools/lr_timeline.py > gpurun_out/lr_timeline.json 2> gpurun_out/lr_timeline.err
GG_LR_TRACE=1 REPS=2 timeout 300 python tools/lr_trace.py > gpurun_out/lr_trace.out 2> gpurun_out/lr_trace.err
exit 0
