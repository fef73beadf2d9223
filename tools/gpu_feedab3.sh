#!/bin/bash
# FEED A/B (tool): e2e / C3 / C4 with paced streaming-store blocks everywhere vs default, interleaved.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2; do
  for cfg in "GG_AB=default" "GG_FEED_NT_ALL=1" "GG_FEED_STATIC=1"; do
    tag=$(echo $cfg | tr ' =' '__')_$rep
    env $cfg timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-l1 --no-ondemand \
      > gpurun_out/fab_$tag.json 2> gpurun_out/fab_$tag.err
  done
done
exit 0
