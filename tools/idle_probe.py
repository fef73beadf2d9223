"""Probe pinned H2D behaviour on the GPU box (tool): clean vs freshly CPU-written buffers."""
import time

import torch

N = 24 << 20
h = torch.empty(N, dtype=torch.uint8).pin_memory()
d = torch.empty_like(h, device="cuda")
s = torch.cuda.Stream()


def timed_copy():
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        d.copy_(h, non_blocking=True)
        e1.record(s)
    e1.synchronize()
    return round(e0.elapsed_time(e1), 3)


print("clean      ", [timed_copy() for _ in range(5)])
hv = h.view(torch.int64)
res = []
for i in range(5):
    hv.fill_(i)              # CPU writes the whole buffer (single thread)
    res.append(timed_copy())
print("cpu-written", res)
res = []
for i in range(5):
    hv.copy_(torch.randint(0, 1 << 62, (N // 8,)))   # CPU writes via a copy
    res.append(timed_copy())
print("cpu-copied ", res)
