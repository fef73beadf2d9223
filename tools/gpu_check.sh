#!/bin/bash
# One GPU session: environment facts, GPU tests, smoke, bench, launch list, ncu capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
{ nvidia-smi; nproc; lscpu | head -20; free -g; } > gpurun_out/box.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=40 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 python bench.py --workload c5 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
[ -x tools/step_bench ] && timeout 300 tools/step_bench > gpurun_out/step_bench.txt 2>&1
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-ondemand --no-apps > gpurun_out/ncu_bench.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:gg_fill64 -s 1 -c 1 -o gpurun_out/prof_fill python tools/prof_fill.py > gpurun_out/ncu_full.log 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:gg_fill_l1 -s 1 -c 1 -o gpurun_out/prof_l1 python tools/prof_l1.py > gpurun_out/ncu_l1.log 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:mc_epoch -s 2 -c 1 -o gpurun_out/prof_mc python tools/prof_mc.py > gpurun_out/ncu_mc.log 2>&1
fi
exit 0
