#!/bin/bash
# GPU session: C5 parity tests + bench --workload c5 (N=1).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_c5.py -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_c5.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_c5.log
timeout 900 python bench.py --workload c5 --no-cpu-baseline ${C5_ARGS} > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
echo "bench rc=$?" >> gpurun_out/bench_c5.err
exit 0
