#!/bin/bash
# GPU session: aligned-table walk -- parity, A/B, ncu, bench (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_table.py tests/test_gpu_variants.py tests/test_gpu_generator.py \
  tests/test_gpu_ondemand.py tests/test_gpu_mc.py tests/test_gpu_example.py tests/test_gpu_fuzz.py -q \
  -p no:cacheprovider --timeout 600 --timeout-method=thread > gpurun_out/pytest_t3.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_t3.log
AB_REPS=3 timeout 900 python tools/ab_fill.py "" "GG_FILL_TABLE=8" "GG_FILL_TABLE=2" "GG_FILL_TABLE=0" > gpurun_out/ab_table4.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gg_fill64 -s 1 -c 1 \
  -o gpurun_out/prof_fill_table python tools/prof_fill.py > gpurun_out/ncu_full.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
exit 0
