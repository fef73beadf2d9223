#!/bin/bash
# GPU session: C3 list ranking with the per-round trace (GG_LR_TRACE=1) (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
GG_LR_TRACE=1 timeout 600 python tools/lr_trace.py > gpurun_out/lr_trace.out 2> gpurun_out/lr_trace.err
