#!/bin/bash
# GPU session: C2 e2e vs ring-slot depth D (draws per streamed slot), interleaved (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for rep in 1 2; do for D in ${DS:-16 8 32 64}; do
  GG_E2E_D=$D timeout 300 python bench.py --no-cpu-baseline --no-l1 --no-apps --no-ondemand --steps 3 --e2e-steps 3 > gpurun_out/e2e_d.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/e2e_d.json').read().strip().splitlines()[-1]); print('D=$D', round(d['e2e']['value'],3))" >> gpurun_out/e2e_slot.txt
done; done
