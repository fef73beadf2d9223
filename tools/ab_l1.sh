#!/bin/bash
# A/B of the l = 1 fill under env configs (tool): median of REPS timed fills each.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for cfg in "$@"; do
  env $cfg REPS=8 python tools/prof_l1.py 2>/dev/null | grep '^ms' | awk '{print $2}' | sort -n | \
    awk -v c="$cfg" '{t[NR]=$1} END{printf "%-30s median %.3f ms\n", c, t[int((NR+1)/2)]}'
done
