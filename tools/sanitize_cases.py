"""Small runs of every kernel family for compute-sanitizer (tool, not product).

    compute-sanitizer --tool memcheck|racecheck|synccheck python tools/sanitize_cases.py
Covers: init, bulk fill (x2 TMA u64/u32, x1 TMA, LDG, generic m, bipartite,
l = 1 TMA; the composed-step table kernels (l = 64 and any l) and, under the hooks, the R2P and
pair kernels), on-demand
consume in every walk mode, list ranking (Phase I-III, the compaction
kernel over several tiles), Monte Carlo epoch.
Sizes are tiny (the sanitizer slows kernels by orders of magnitude) but
ragged: partial units, partial warps, several draws per TMA stage.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

dev = "cuda:0"
W = 200  # 3 full 64-walker units + a ragged one
for kw in ({}, {"m": 256}, {"m": 1000}, {"walk_len": 1}, {"walk_len": 17, "m": 12345},
           {"walk_len": 13}, {"walk_len": 16, "m": 1 << 20}, {"variant": 1}):
    g = Generator(walkers=W, seed=11, **kw)
    o = torch.empty(W * 5 + 7, dtype=torch.int64, device=dev)
    g.fill(o)
    g.prefetch(6)
    g.fill(o[: W * 5])
    if kw.get("m") in (None,):
        o32 = torch.empty(W * 4 * 2, dtype=torch.int32, device=dev)
        g.fill(o32)
    torch.cuda.synchronize()
    g.close()
print("fill ok")

# on demand, one generator per walk mode (prng_walk_mode: l = 64 pow2, its
# bipartite form, any l pow2, l = 64 with m <= 2^30, generic)
for kw in ({}, {"variant": 1}, {"walk_len": 17}, {"m": 1000}, {"m": (1 << 32) - 5}):
    g = Generator(walkers=W, seed=12, **kw)
    g.epoch_begin(W, 5)
    o = torch.empty(W * 5, dtype=torch.int64, device=dev)
    g.consume(W, uniform=5, out=o)
    g.epoch_end()
    torch.cuda.synchronize()
    g.close()
print("consume ok")

n = 10000  # several compaction tiles (2048 items each) per round
succ, pred, head = inputs.random_list(n, 5)
g = Generator(walkers=n, seed=13)
r, info = g.list_rank(torch.from_numpy(succ).to(dev), torch.from_numpy(pred).to(dev), head)
torch.cuda.synchronize()
assert int(r[head].item()) == 0
g.close()
print("list ranking ok", info["rounds"])

layers = ((1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2))
g = Generator(walkers=256, seed=14)
res = g.mc_run(layers, photons_total=512, threads=256, epoch_draws=48)
torch.cuda.synchronize()
g.close()
print("mc ok", res["draws"])
