#!/bin/bash
# Battery on the f1 / f3 variants (tool): bipartite walk at 2^36 words, rand_r seed bits at 2^33.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1500 python tools/battery_big.py --streams 5 --log2-words-extra 36 > gpurun_out/battery_bip.json 2> gpurun_out/battery_bip.err
timeout 1500 python tools/battery_big.py --streams 6 --log2-words-extra 33 > gpurun_out/battery_randr.json 2> gpurun_out/battery_randr.err
exit 0
