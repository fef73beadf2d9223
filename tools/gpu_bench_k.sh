#!/bin/bash
# GPU session: K-mode bench only (fill + l=1 + on-demand), interleaved A/B of the fill.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
AB_REPS=${AB_REPS:-3} timeout 900 python tools/ab_fill.py "" ${AB_CONFIGS} > gpurun_out/ab.txt 2>&1
timeout 600 python bench.py --no-e2e --no-apps --no-cpu-baseline > gpurun_out/bench_k.json 2> gpurun_out/bench_k.err
exit 0
