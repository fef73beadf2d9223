#!/bin/bash
# A/B of the e2e fill under feed variants (tool): env configs as arguments,
#   bash tools/ab_e2e.sh "" "GG_FEED_NT_ALL=1" "GG_FEED_CHUNK_MB=64"
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
[ $# -eq 0 ] && set -- "" "GG_FEED_NO_NT=1"
for rep in 1 2; do
  i=0
  for cfg in "$@"; do
    i=$((i+1))
    env $cfg python bench.py --no-cpu-baseline --no-l1 --no-apps --no-ondemand --steps 3 --e2e-steps 4 > gpurun_out/e2e_$i.$rep.json 2>/dev/null
    python -c "import json; d=json.loads(open('gpurun_out/e2e_$i.$rep.json').read().strip().splitlines()[-1]); print(repr('$cfg'), round(d['e2e']['value'],3), round(d['e2e']['feed_s_per_step'],3))"
  done
done
