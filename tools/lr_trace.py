"""Per-round timing of gg_list_rank at 2^24 nodes (tool): GG_LR_TRACE=1 [HOST_THREADS=k] python tools/lr_trace.py"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

n = 1 << 24
succ, pred, head = inputs.random_list(n, 0x5EED0003)
s, p = torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda()
for rep in range(int(os.environ.get("REPS", "3"))):
    g = Generator(walkers=n, seed=0x5EED0003, host_threads=int(os.environ.get("HOST_THREADS", "0")))
    torch.cuda.synchronize()
    t = time.perf_counter()
    rank, info = g.list_rank(s, p, head)
    torch.cuda.synchronize()
    print("wall ms", (time.perf_counter() - t) * 1e3, info, file=sys.stderr)
    g.close()
