#!/bin/bash
# Round-2 GPU session C: FEED experiments (second copy stream, write-combined chunks) (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_variants.py -q -p no:cacheprovider -k "FEED" > gpurun_out/variants.log 2>&1
timeout 900 python tools/lr_feed_probe.py "" "GG_FEED_STREAMS=2" "GG_FEED_WC=1" "GG_FEED_STREAMS=2 GG_FEED_WC=1" \
  "HOST_THREADS=8 GG_FEED_STREAMS=2" "GG_FEED_STREAMS=2 GG_FEED_CHUNKS=6" > gpurun_out/lr_feed_probe2.json 2> gpurun_out/lr_feed_probe2.err
timeout 1200 bash tools/ab_e2e.sh "" "GG_FEED_STREAMS=2" "GG_FEED_WC=1" "GG_FEED_STREAMS=2 GG_FEED_WC=1" > gpurun_out/ab_e2e.txt 2>&1
exit 0
