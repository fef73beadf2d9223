"""K-mode fill time for small N (tool; Fig. 3's low end): python tools/small_n_ab.py
(hooks such as GG_FILL_KPW from the environment).  Prints one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W = 1 << 20
res = {"env": {k: v for k, v in os.environ.items() if k.startswith("GG_")}}
g = Generator(walkers=W, seed=0x5EED0002)
g.prefetch(96)
g.mark()
out = torch.empty(W * 96, dtype=torch.int64, device="cuda")
for n_m in (5, 10, 50, 100):
    n = n_m * 1000 * 1000
    ts = []
    for rep in range(6):
        g.rewind()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        g.fill(out[:n])
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    res[f"N{n_m}M_gnum_s"] = round(n / (min(ts[1:]) / 1e3) / 1e9, 2)
print(json.dumps(res))
