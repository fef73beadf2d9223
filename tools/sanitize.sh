#!/bin/bash
# GPU session: compute-sanitizer memcheck / racecheck / synccheck / initcheck on small runs of every kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > gpurun_out/san_$tool.txt 2>&1
  echo "rc=$?" >> gpurun_out/san_$tool.txt
done
# the pair fill variants (hook read once per process)
for pair in 1 3 4; do for tool in memcheck racecheck synccheck; do
  GG_FILL_PAIR=$pair timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py \
    > gpurun_out/san_pair${pair}_$tool.txt 2>&1
  echo "rc=$?" >> gpurun_out/san_pair${pair}_$tool.txt
done; done
exit 0
