#!/bin/bash
# GPU session: ORB table layout -- full GPU tests, A/B, ncu, bench (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 --timeout-method=thread \
  --durations=10 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
AB_REPS=3 timeout 900 python tools/ab_fill.py "" "GG_FILL_ORB=0" "GG_FILL_TABLE=8" "GG_FILL_TABLE=0" > gpurun_out/ab_table5.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gg_fill64 -s 1 -c 1 \
  -o gpurun_out/prof_fill_table python tools/prof_fill.py > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ondemand --no-apps > gpurun_out/ncu_bench.log 2>&1
timeout 600 python tools/variant_probe.py > gpurun_out/variants.json 2> gpurun_out/variants.err
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
exit 0
