#!/bin/bash
# Short GPU session: selected tests + microbenchmark.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest ${TESTS:-tests} -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
[ -x tools/step_bench ] && timeout 300 tools/step_bench > gpurun_out/step_bench.txt 2>&1
[ -n "$BENCH" ] && timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
exit 0
