#!/bin/bash
# C3 pace-rate A/B (tool): GG_FEED_RATE in GB/s, interleaved; lr_trace prints per-call wall ms.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out; : > gpurun_out/rate_ab.txt
for rep in 1 2 3; do for r in 52 56 60 64 68; do
  echo "rate $r" >> gpurun_out/rate_ab.txt
  GG_FEED_RATE=$r REPS=4 timeout 300 python tools/lr_trace.py 2>&1 | grep "wall ms" | cut -c1-30 >> gpurun_out/rate_ab.txt
done; done
exit 0
