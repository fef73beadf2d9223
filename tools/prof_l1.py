"""Profile target: the l = 1 fill (f1) as bench.py runs it (2^20 walkers x 1024 draws).

    ncu --set full -k regex:gg_fill_l1 -s 1 -c 1 python tools/prof_l1.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W, D = 1 << 20, 1024
g = Generator(walkers=W, seed=0x5EED0002, walk_len=1)
g.prefetch(D)
g.mark()
out = torch.empty(W * D, dtype=torch.int64, device="cuda")
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
for i in range(int(os.environ.get("REPS", "3"))):
    g.rewind()
    ev[0].record()
    g.fill(out)
    ev[1].record()
    torch.cuda.synchronize()
    print("ms", ev[0].elapsed_time(ev[1]), "GB/s", W * D * 12 / ev[0].elapsed_time(ev[1]) / 1e6)
