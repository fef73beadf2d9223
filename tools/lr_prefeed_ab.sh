#!/bin/bash
# GPU session: list-ranking parity + C3 wall time with / without the next-round prefeed (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_listrank.py tests/test_gpu_ondemand.py -m gpu -q -x -p no:cacheprovider > gpurun_out/pylr2.log 2>&1
echo rc=$? >> gpurun_out/pylr2.log
for rep in 1 2; do for cfg in "GG_LR_PREFEED=0" "GG_LR_PREFEED=1"; do
  echo "cfg [$cfg]" >> gpurun_out/lr_pf.txt
  env $cfg REPS=4 timeout 300 python tools/lr_trace.py 2>&1 | grep "wall ms" | cut -c1-24 | tail -3 | tr '\n' ' ' >> gpurun_out/lr_pf.txt
  echo >> gpurun_out/lr_pf.txt
done; done
