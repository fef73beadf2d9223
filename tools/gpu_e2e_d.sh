#!/bin/bash
# e2e ring-slot depth A/B (tool), interleaved x4.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2 3 4; do for d in 4 8 16; do
  GG_E2E_D=$d timeout 600 python bench.py --steps 3 --warmup 3 --e2e-steps 3 --no-cpu-baseline --no-l1 --no-ondemand --no-apps \
    > gpurun_out/e2ed_${d}_$rep.json 2> gpurun_out/e2ed_${d}_$rep.err
done; done
exit 0
