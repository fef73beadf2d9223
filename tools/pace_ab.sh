#!/bin/bash
# GPU session (tool): full bench with the paced FEED (default) vs the round-1
# FEED (unpaced), interleaved twice.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2; do
  for cfg in "GG_AB=paced" "GG_FEED_RATE=0"; do
    tag=$(echo $cfg | tr ' =' '__')_$rep
    env $cfg timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-l1 --no-ondemand \
      > gpurun_out/pab_$tag.json 2> gpurun_out/pab_$tag.err
  done
done
