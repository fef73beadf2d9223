#!/bin/bash
# Round-2 GPU session D: SM-driven TRANSFER (GG_FEED_PULL=1) vs the copy engine (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_variants.py -q -p no:cacheprovider -k "PULL" > gpurun_out/variants.log 2>&1
timeout 900 python tools/lr_feed_probe.py "" "GG_FEED_PULL=1" "GG_FEED_PULL=1 HOST_THREADS=12" > gpurun_out/lr_feed_probe3.json 2> gpurun_out/lr_feed_probe3.err
timeout 1200 bash tools/ab_e2e.sh "" "GG_FEED_PULL=1" > gpurun_out/ab_e2e_pull.txt 2>&1
exit 0
