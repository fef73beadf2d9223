cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_generator.py tests/test_gpu_fuzz.py tests/test_gpu_edges.py -m gpu -q -x -p no:cacheprovider > gpurun_out/pyl1.log 2>&1; echo rc=$? >> gpurun_out/pyl1.log
for rep in 1 2; do for cfg in "GG_L1_TMA_STORE=0" "GG_L1_TMA_STORE=1"; do
  env $cfg timeout 300 python bench.py --no-e2e --no-apps --no-ondemand --no-cpu-baseline --steps 10 > gpurun_out/l1.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/l1.json').read().strip().splitlines()[-1]); print('$cfg', round(d['l1_fill']['value'],1), round(d['l1_fill']['roofline']['frac'],3), round(d['l1_fill']['ms_kernel'],3))" >> gpurun_out/l1ab.txt
done; done
