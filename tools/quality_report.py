"""Battery report on GPU output (tool, Tables II-III):
tests/battery.py (+ the Crush-style tests of tests/battery_crush.py) on 2^24 labels (2^25 u32 words) of the C2 generator, in bulk
and walker-major order, for l = 64 (the paper's walk), l = 16 and l = 1.

    python tools/quality_report.py > profiles/r01_battery.json
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import battery as B  # noqa: E402
import battery_crush as C  # noqa: E402
from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W, D = 1 << 18, 64
rep = {"config": f"m=2^32, l0=64, seed 0x5EED0002, {W} walkers x {D} draws = 2^24 labels "
                 "(2^25 u32 words, R12) per order", "alpha_per_test": 1e-4, "runs": {}}
for l in (64, 16, 1):
    g = Generator(walkers=W, seed=0x5EED0002, walk_len=l)
    o = torch.empty(W * D, dtype=torch.int64, device="cuda")
    g.fill(o)
    z = o.cpu().numpy().view(np.uint64).reshape(D, W)
    g.close()
    for order, arr in (("bulk", z), ("walker-major", z.T)):
        t = time.time()
        words = np.ascontiguousarray(arr).reshape(-1).view(np.uint32)
        res = B.run(words)
        res.update({f"crush:{k}": v for k, v in C.run(words).items()})
        rep["runs"][f"l={l} {order}"] = {
            "p": {k: float(f"{v:.3g}") for k, v in res.items()},
            "failed": sorted(k for k, v in res.items() if v < 1e-4),
            "seconds": round(time.time() - t, 1)}
print(json.dumps(rep, indent=1))
