"""FEED generation rate by window shape (tool): prefetch of D draws for W walkers,
host threads = all cores; gen GB/s = bits fed / time inside the feed thread pool,
prefetch GB/s = bits fed / wall time of prng_prefetch (feed + H2D overlapped)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

for W, D in ((1 << 20, 64), (1 << 22, 16), (1 << 23, 8), (1 << 20, 512)):
    for rep in range(2):
        g = Generator(walkers=W, seed=1)
        s0 = g.stats()
        t = time.perf_counter()
        g.prefetch(D)
        wall = time.perf_counter() - t
        s = g.stats()
        fed = s["bits_bytes_fed"] - s0["bits_bytes_fed"]
        print(f"W=2^{W.bit_length()-1} D={D}: {fed/1e9:.2f} GB, gen {fed/(s['feed_seconds']-s0['feed_seconds'])/1e9:.1f} GB/s, "
              f"prefetch {fed/wall/1e9:.1f} GB/s", flush=True)
        g.close()
