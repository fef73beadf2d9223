#!/bin/bash
# A/B of the e2e fill with and without non-temporal feed stores (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2; do
  for mode in nt cached; do
    if [ $mode = cached ]; then export GG_FEED_NO_NT=1; else unset GG_FEED_NO_NT; fi
    python bench.py --no-cpu-baseline --no-l1 --no-apps --no-ondemand --steps 3 --e2e-steps 3 > gpurun_out/e2e_$mode.$rep.json 2>/dev/null
    python -c "import json; d=json.load(open('gpurun_out/e2e_$mode.$rep.json')); print('$mode', round(d['e2e']['value'],3), round(d['e2e']['feed_s_per_step'],3))"
  done
done
