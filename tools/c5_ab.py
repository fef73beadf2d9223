"""A/B of the C5-shaped K-mode fill (tool): 2^23 walkers x 32 draws per call.

    python tools/c5_ab.py "" "GG_FILL_KPW=2" "GG_FILL_TABLE=8" ...

Each config (env assignments) runs in its own process: one Generator of 2^23
walkers, the 32-draw window prefetched, then REPS x (rewind + prng_fill of
2^28 labels), device-timed (AB_W / AB_D override the shape; AB_FRESH=1
prefetches a new window before every fill, as the C5 bench does) with CUDA events; prints the median ms and G
labels/s per config.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, json, os
sys.path.insert(0, %(root)r)
import torch
from paper_conf_ipps_banerjeebk12_b200 import Generator
W, D = int(os.environ.get("AB_W", 1 << 23)), int(os.environ.get("AB_D", 32))
g = Generator(walkers=W, seed=0x5EED0005)
g.prefetch(D)
g.mark()
out = torch.empty(W * D, dtype=torch.int64, device="cuda")
ms = []
fresh = os.environ.get("AB_FRESH") == "1"  # C5's order: prefetch the next window, then fill it
warm = torch.randn(2048, 2048, device="cuda") * 0.01 if os.environ.get("AB_WARM") == "1" else None
for i in range(12):
    if fresh:
        g.prefetch(D)
    else:
        g.rewind()
    if warm is not None:  # diagnostic: keep the SMs busy ~5 ms right before the timed fill
        for _ in range(20):
            warm = warm @ warm
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); g.fill(out); b.record(); torch.cuda.synchronize()
    if i >= 2:
        ms.append(a.elapsed_time(b))
ms.sort()
print(json.dumps({"ms_median": ms[len(ms) // 2], "ms_min": ms[0], "G_per_s": W * D / ms[len(ms) // 2] / 1e6}))
"""


def main():
    res = {}
    for c in sys.argv[1:] or [""]:
        env = dict(os.environ)
        for kv in c.split():
            k, v = kv.split("=")
            env[k] = v
        p = subprocess.run([sys.executable, "-c", CHILD % {"root": ROOT}], env=env,
                           capture_output=True, text=True, timeout=600)
        res[c or "default"] = (json.loads(p.stdout.strip().splitlines()[-1]) if p.returncode == 0
                               else {"error": p.stderr[-400:]})
        print(c or "default", res[c or "default"], file=sys.stderr)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
