#!/bin/bash
# GPU session: step-formulation microbenchmark + pipe counters (tool, not product).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 tools/step_bench2 5 > gpurun_out/step_bench2.txt 2>&1
timeout 600 ncu --clock-control none -k regex:kfill2 -c 4 --metrics \
  smsp__inst_executed.sum,sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_fmalite.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed_pipe_xu.sum,sm__inst_executed_pipe_uniform.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum \
  --csv tools/step_bench2 1 > gpurun_out/step_bench2_ncu.csv 2>&1
exit 0
