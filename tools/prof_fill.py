"""Profile target: one warm-up + one timed bulk prng_fill of the C2 workload.

    ncu --set full -k regex:gg_fill64 -s 1 -c 1 python tools/prof_fill.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W = 1 << 20
g = Generator(walkers=W, seed=0x5EED0002)
draws = int(os.environ.get("DRAWS", "512"))
g.prefetch(draws)
g.mark()
out = torch.empty(W * draws * 2, dtype=torch.int32, device="cuda")
for _ in range(int(os.environ.get("REPS", "2"))):
    g.rewind()
    g.fill(out)
torch.cuda.synchronize()
print("ok", out[:4].tolist())
