#!/bin/bash
# GPU session: table walk in the on-demand consumers -- parity, MC register budget A/B, bench (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_ondemand.py tests/test_gpu_mc.py tests/test_gpu_listrank.py \
  tests/test_gpu_example.py tests/test_gpu_variants.py tests/test_gpu_table.py tests/test_gpu_fuzz.py -q \
  -p no:cacheprovider --timeout 600 --timeout-method=thread > gpurun_out/pytest_t2.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_t2.log
for minb in 8 6 4; do
  GG_MC_MINB=$minb timeout 600 python tools/prof_mc.py > gpurun_out/mc_minb$minb.txt 2>&1
done
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
exit 0
