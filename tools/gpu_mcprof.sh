#!/bin/bash
# MC epoch kernel ncu capture (table walk) + a repeat bench line (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 300 python tools/prof_mc.py > gpurun_out/prof_mc_plain.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mc_epoch -s 3 -c 1 \
  -o gpurun_out/prof_mc_table python tools/prof_mc.py > gpurun_out/ncu_mc.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_rep.json 2> gpurun_out/bench_rep.err
exit 0
