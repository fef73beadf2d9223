#!/bin/bash
# GPU session: feed-thread pinning A/B (GG_FEED_PIN=1) on C2 e2e and C3 list ranking (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
{ nvidia-smi topo -m; B=$(nvidia-smi --query-gpu=pci.bus_id --format=csv,noheader | head -1 | tr 'A-F' 'a-f' | sed 's/^00000000/0000/'); echo "bus $B"; cat /sys/bus/pci/devices/$B/local_cpulist; cat /sys/bus/pci/devices/$B/numa_node; lscpu | grep -i "numa\|socket\|core\|thread"; } > gpurun_out/pin_topo.txt 2>&1
for rep in 1 2; do for cfg in "" "GG_FEED_PIN=1"; do
  env $cfg timeout 300 python bench.py --no-cpu-baseline --no-l1 --no-ondemand --steps 3 --e2e-steps 3 > gpurun_out/pin.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/pin.json').read().strip().splitlines()[-1]); print(repr('$cfg'), 'e2e', round(d['e2e']['value'],3), 'lr_ms', round(d['apps']['list_ranking']['ms_wall'],1), 'mc_ms', round(d['apps']['monte_carlo']['ms_wall']))" >> gpurun_out/pin_ab.txt
done; done
