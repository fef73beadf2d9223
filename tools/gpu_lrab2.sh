#!/bin/bash
# C3 FEED A/B session 2 (tool): speculative prefeed bound, pace rate.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_variants.py tests/test_gpu_listrank.py -q -p no:cacheprovider \
  > gpurun_out/pytest_var.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_var.log
timeout 300 python tools/lr_timeline.py > gpurun_out/lr_timeline.json 2> gpurun_out/lr_timeline.err
timeout 1500 python tools/feed_ab.py --reps 3 "" "GG_LR_PREFEED=2" "GG_FEED_RATE=60" "GG_FEED_RATE=80" \
  > gpurun_out/feed_ab.json 2> gpurun_out/feed_ab.err
exit 0
