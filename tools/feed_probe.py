"""Probe FEED + TRANSFER rates (tool): epoch windows of A walkers x 1 draw vs raw H2D."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W = 1 << 24
g = Generator(walkers=W, seed=1)
s = torch.cuda.current_stream()
for A in (16_777_216, 8_000_000, 3_376_777, 1_000_000, 3_376_800):
    for rep in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        g.epoch_begin(A, 1)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        g.epoch_end()
        mb = A * 24 / 1e6
        print(f"A={A:>9} {mb:7.1f} MB  feed+enqueue {1e3*(t1-t0):7.3f} ms  copy tail {1e3*(t2-t1):7.3f} ms"
              f"  -> {mb/1e3/(t2-t0):6.1f} GB/s", flush=True)
for mb in (27, 81, 400):
    h = torch.empty(mb * 1 << 20, dtype=torch.uint8).pin_memory()
    d = torch.empty_like(h, device="cuda")
    for rep in range(3):
        torch.cuda.synchronize()
        t = time.perf_counter()
        d.copy_(h, non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
        print(f"raw pinned H2D {mb} MiB: {dt*1e3:.3f} ms -> {mb*1.048576/1e3/dt:.1f} GB/s", flush=True)
print(g.stats())

# pointer attributes of the library's pinned chunks (are they registered?)
import ctypes  # noqa: E402
