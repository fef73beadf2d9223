#!/bin/bash
# GPU session: compute-sanitizer memcheck / racecheck / synccheck / initcheck on small runs of every kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > gpurun_out/san_$tool.txt 2>&1
  echo "rc=$?" >> gpurun_out/san_$tool.txt
done
# the R2P fill kernels, the plain table layout and the pair variant (hooks read once per process)
for cfg in "GG_FILL_TABLE=0" "GG_FILL_ORB=0" "GG_FILL_TABLE=8" "GG_FILL_TABLE=0 GG_FILL_PAIR=1"; do
  tag=$(echo $cfg | tr ' =' '__')
  for tool in memcheck racecheck synccheck; do
    env $cfg timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py \
      > gpurun_out/san_${tag}_$tool.txt 2>&1
    echo "rc=$?" >> gpurun_out/san_${tag}_$tool.txt
  done
done
exit 0
