#!/bin/bash
# MC epoch kernel blocks-per-SM A/B (tool): in-kernel time of the C4 run.
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out; : > gpurun_out/mcminb.txt
for rep in 1 2; do for m in 4 6 8 12; do
  echo "minb $m $(GG_MC_MINB=$m timeout 300 python tools/prof_mc.py 2>&1 | tail -1)" >> gpurun_out/mcminb.txt
done; done
exit 0
