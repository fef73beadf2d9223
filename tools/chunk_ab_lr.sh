#!/bin/bash
# GPU session: C3 wall time vs pinned chunk size / count (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2; do for cfg in "" "GG_FEED_CHUNK_MB=32" "GG_FEED_CHUNK_MB=8 GG_FEED_CHUNKS=8" "GG_FEED_CHUNKS=8" "GG_FEED_CHUNK_MB=64"; do
  echo "cfg [$cfg]" >> gpurun_out/chk.txt
  env $cfg REPS=4 timeout 300 python tools/lr_trace.py 2>&1 | grep "wall ms" | cut -c1-24 | tail -3 | tr '\n' ' ' >> gpurun_out/chk.txt
  echo >> gpurun_out/chk.txt
done; done
