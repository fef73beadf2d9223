#!/bin/bash
# C4 FEED A/B (tool): epoch windows streamed (default) vs cached (>= 1 GB), interleaved x4.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2 3 4; do
  for cfg in "GG_AB=default" "GG_FEED_EPOCH_CACHED=1"; do
    tag=$(echo $cfg | tr ' =' '__')_$rep
    env $cfg timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-l1 --no-ondemand --no-e2e \
      > gpurun_out/mab_$tag.json 2> gpurun_out/mab_$tag.err
  done
done
exit 0
