#!/bin/bash
# GPU session: three default bench runs back to back (run-to-run spread) (tool).
cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
for i in 1 2 3; do timeout 900 python bench.py --no-cpu-baseline > gpurun_out/rep_$i.json 2>/dev/null; done
python - <<'PY'
import json
rows = []
for i in (1, 2, 3):
    d = json.loads(open(f"gpurun_out/rep_{i}.json").read().strip().splitlines()[-1])
    rows.append({"value": d["value"], "frac": d["roofline"]["frac"], "kernel_ms": d["roofline"]["kernel_ms"],
                 "e2e": d["e2e"]["value"], "e2e_frac_of_pcie_bound": d["e2e"].get("bound", {}).get("frac"),
                 "on_demand_uniform": d["on_demand"]["uniform_S100"], "l1": d["l1_fill"]["value"],
                 "c3_ms": d["apps"]["list_ranking"]["ms_wall"], "c4_ms": d["apps"]["monte_carlo"]["ms_wall"],
                 "sm_mhz": d["clocks"]["sm_mhz"], "reasons": d["clocks"]["reasons"]})
json.dump(rows, open("gpurun_out/bench_repeats.json", "w"), indent=1)
print(json.dumps(rows, indent=1))
PY
