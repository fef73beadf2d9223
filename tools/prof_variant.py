"""Profile target (tool): K-mode fill of a walk variant, 2^20 walkers x 64 draws.

    VARIANT=1 ncu --set full -k regex:gg_fill64x2 -s 1 -c 1 python tools/prof_variant.py
    (VARIANT=1 bipartite; M=... for another modulus; L=... for another walk length)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W, D = 1 << 20, 64
g = Generator(walkers=W, seed=9, variant=int(os.environ.get("VARIANT", "1")),
              m=int(os.environ.get("M", str(1 << 32))), walk_len=int(os.environ.get("L", "64")))
g.prefetch(D)
g.mark()
o = torch.empty(W * D, dtype=torch.int64, device="cuda")
for _ in range(2):
    g.rewind()
    g.fill(o)
torch.cuda.synchronize()
print("ok")
