#!/bin/bash
# Round-2 GPU session: full GPU tests (per-test timeout), smoke, fill A/B, bench (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
{ nvidia-smi; nproc; free -g; } > gpurun_out/box.txt 2>&1
timeout 3000 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 900 --timeout-method=thread \
  --durations=40 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
AB_REPS=3 timeout 900 python tools/ab_fill.py "" "GG_FILL_PAIR=1" "GG_FILL_PAIR=2" > gpurun_out/ab_fill.txt 2>&1
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
exit 0
