#!/bin/bash
# BigCrush-volume battery session (tool): 2^38 words per l = 64 stream.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 3300 python tools/battery_big.py --log2-words 38 > gpurun_out/battery38.json 2> gpurun_out/battery38.err
echo "rc=$?" >> gpurun_out/battery38.err
exit 0
