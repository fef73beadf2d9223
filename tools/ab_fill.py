"""Interleaved A/B timing of the bulk fill under different env configs (tool).

    python tools/ab_fill.py "GG_FILL_MINB=24" "GG_FILL_KPW=2" ...
Each config runs in its own subprocess (env is read once per process);
configs are interleaved R times; prints the median kernel ms per config.
"""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
configs = sys.argv[1:] or [""]
R = int(os.environ.get("AB_REPS", "3"))
res = {c: [] for c in configs}
for r in range(R):
    for c in configs:
        env = dict(os.environ)
        for kv in c.split():
            k, v = kv.split("=")
            env[k] = v
        out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--no-e2e",
                              "--no-cpu-baseline", "--no-ondemand", "--no-apps", "--steps", "20"],
                             env=env, capture_output=True, text=True, timeout=600)
        d = json.loads(out.stdout.strip().splitlines()[-1])
        res[c].append(d["roofline"]["kernel_ms"])
for c, v in res.items():
    print(f"{c or 'default':30s} median {statistics.median(v):.3f} ms  all {[round(x, 3) for x in v]}")
