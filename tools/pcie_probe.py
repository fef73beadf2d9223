"""Diagnostic (tool): raw pinned H2D / D2H rates on this box (torch copies,
CUDA events): one stream vs two concurrent streams, several chunk sizes.

    python tools/pcie_probe.py
"""
import json

import torch

res = {}
dev = torch.device("cuda", 0)
big = 1 << 30
h = torch.empty(big, dtype=torch.uint8).pin_memory()
d = torch.empty(big, dtype=torch.uint8, device=dev)
h.fill_(1)
s = [torch.cuda.Stream(), torch.cuda.Stream()]


def timed(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(torch.cuda.current_stream())
        fn()
        for st in s:
            torch.cuda.current_stream().wait_stream(st)
        e1.record(torch.cuda.current_stream())
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


for chunk_mb in (4, 32, 128, 1024):
    c = chunk_mb << 20
    n = big // c

    def one():
        for i in range(n):
            d[i * c:(i + 1) * c].copy_(h[i * c:(i + 1) * c], non_blocking=True)

    def two():
        for i in range(n):
            with torch.cuda.stream(s[i & 1]):
                d[i * c:(i + 1) * c].copy_(h[i * c:(i + 1) * c], non_blocking=True)

    def d2h():
        for i in range(n):
            h[i * c:(i + 1) * c].copy_(d[i * c:(i + 1) * c], non_blocking=True)

    def both():
        half = big // 2
        with torch.cuda.stream(s[0]):
            d[:half].copy_(h[:half], non_blocking=True)
        with torch.cuda.stream(s[1]):
            h[half:].copy_(d[half:], non_blocking=True)

    res[f"h2d_{chunk_mb}MB_1stream_GBs"] = big / timed(one) / 1e6
    if n > 1:
        res[f"h2d_{chunk_mb}MB_2streams_GBs"] = big / timed(two) / 1e6
    res[f"d2h_{chunk_mb}MB_GBs"] = big / timed(d2h) / 1e6
res["bidirectional_512MB_each_GBs_total"] = big / timed(lambda: None or None) if False else None
half = big // 2


def both():
    with torch.cuda.stream(s[0]):
        d[:half].copy_(h[:half], non_blocking=True)
    with torch.cuda.stream(s[1]):
        h[half:].copy_(d[half:], non_blocking=True)


res["bidirectional_total_GBs"] = big / timed(both) / 1e6
print(json.dumps(res, indent=1))
