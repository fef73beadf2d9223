"""Fill time per label vs walker count (tool): shows the cost of the last partial
round of 64-walker units (C2 has 16384 units for ~5328 resident warps).

    python tools/tail_probe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

D = 512
for W in [1 << 20, 5328 * 64 * 3, 5328 * 64 * 2, 5328 * 64 * 3 + 64 * 148, 5328 * 64 * 3 + 64 * 1332]:
    g = Generator(walkers=W, seed=0x5EED0002)
    g.prefetch(D)
    g.mark()
    out = torch.empty(W * D * 2, dtype=torch.int32, device="cuda")
    ts = []
    for r in range(6):
        g.rewind()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.fill(out)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = sorted(ts[1:])[len(ts[1:]) // 2]
    print(f"W={W:8d} units={W // 64:6d} rounds={W / 64 / 5328:5.2f}  {ms:7.3f} ms  "
          f"{W * D / ms / 1e6:6.2f} G labels/s", flush=True)
    g.close()
    del out
    torch.cuda.empty_cache()
