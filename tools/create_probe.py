"""prng_create (Alg.1: FEED + H2D of 32 B per walker, burn-in kernel) wall time (tool).

    python tools/create_probe.py        -> median of 3 creations at 2^20 and 2^24 walkers
"""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

Generator(walkers=1 << 16, seed=1).close()  # warm (CUDA context, feed threads)
for W in (1 << 20, 1 << 24):
    ts = []
    for r in range(3):
        torch.cuda.synchronize()
        t = time.perf_counter()
        g = Generator(walkers=W, seed=0x5EED0003 + r)
        torch.cuda.synchronize()
        ts.append((time.perf_counter() - t) * 1e3)
        g.close()
    print(f"walkers 2^{W.bit_length() - 1}: prng_create median {statistics.median(ts):.1f} ms "
          f"(all {[round(x, 1) for x in ts]}; {W * 32 / 1e6:.0f} MB of seed bits)")
