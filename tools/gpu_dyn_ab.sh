#!/bin/bash
# e2e A/B (tool): cached-store bulk feed in shared-counter blocks (GG_FEED_DYN_ALL=1) vs per-thread slices, x4.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2 3 4; do for cfg in "GG_AB=default" "GG_FEED_DYN_ALL=1"; do
  tag=$(echo $cfg | tr ' =' '__')_$rep
  env $cfg timeout 600 python bench.py --steps 3 --warmup 3 --e2e-steps 3 --no-cpu-baseline --no-l1 --no-ondemand --no-apps \
    > gpurun_out/dyn_$tag.json 2> gpurun_out/dyn_$tag.err
done; done
exit 0
