"""Throughput of the walk variants (tool): forward maps (R2),
bipartite sigma / sigma^-1 alternation (variant 1), a non-power-of-two m, and
l = 16, each a K-mode fill of 2^20 walkers x 64 draws with the bits resident."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W, D = 1 << 20, 64
res = {}
for name, kw in (("forward m=2^32 l=64", {}), ("bipartite m=2^32 l=64", {"variant": 1}),
                 ("forward m=2^32-5 l=64", {"m": (1 << 32) - 5}),
                 ("forward m=2^30-35 l=64", {"m": (1 << 30) - 35}),
                 ("forward m=2^32 l=16", {"walk_len": 16})):
    g = Generator(walkers=W, seed=9, **kw)
    g.prefetch(D)
    g.mark()
    o = torch.empty(W * D, dtype=torch.int64, device="cuda")
    for _ in range(2):
        g.rewind()
        g.fill(o)
    ts = []
    for _ in range(5):
        g.rewind()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.fill(o)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = sorted(ts)[2]
    res[name] = {"ms": ms, "G_labels_per_s": W * D / ms / 1e6}
    g.close()
print(json.dumps(res, indent=1))
