#!/bin/bash
# C3 FEED A/B session (tool): dynamic paced blocks vs static slices, timeline.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 300 python tools/lr_timeline.py > gpurun_out/lr_timeline.json 2> gpurun_out/lr_timeline.err
GG_FEED_STATIC=1 timeout 300 python tools/lr_timeline.py > gpurun_out/lr_timeline_static.json 2>> gpurun_out/lr_timeline.err
timeout 1200 python tools/feed_ab.py --reps 3 "" "GG_FEED_STATIC=1" > gpurun_out/feed_ab.json 2> gpurun_out/feed_ab.err
exit 0
