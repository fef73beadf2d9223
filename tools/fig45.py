"""Fig.4 / Fig.5 analogues on B200 (§IV-A).

Fig.4: time per number of the three work units FEED (host threads generate
bits), TRANSFER (H2D), GENERATE (walk kernel), and the overlapped E-mode
total, for the C2 generator (m = 2^32, l = 64, 2^20 walkers).
Fig.5: E-mode time vs batch size -- the paper's S (numbers per thread per
launch) is our epoch depth D (draws per walker per streamed ring slot).

    python tools/fig45.py > profiles/r01_fig45.json
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

W = 1 << 20
SEED = 0x5EED0002
out = {"config": "m=2^32, l=l0=64, 2^20 walkers, device output (prng_fill), 24 B of bits per number"}

# GENERATE: walk kernel with resident bits
g = Generator(walkers=W, seed=SEED)
D = 128
g.prefetch(D)
g.mark()
o = torch.empty(W * D, dtype=torch.int64, device="cuda")
for _ in range(3):
    g.rewind()
    g.fill(o)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
g.rewind()
e0.record()
g.fill(o)
e1.record()
torch.cuda.synchronize()
gen_ns = e0.elapsed_time(e1) * 1e6 / (W * D)
# FEED + TRANSFER: prefetch (host generation into pinned chunks + H2D)
s0 = g.stats()
torch.cuda.synchronize()
t = time.perf_counter()
g.prefetch(D)
torch.cuda.synchronize()
pf_s = time.perf_counter() - t
s1 = g.stats()
feed_ns = (s1["feed_seconds"] - s0["feed_seconds"]) * 1e9 / (W * D)
xfer_total_ns = pf_s * 1e9 / (W * D)
g.close()
del o
torch.cuda.empty_cache()

# raw pinned H2D rate for the TRANSFER unit alone
h = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
d = torch.empty_like(h, device="cuda")
for _ in range(3):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
t = time.perf_counter()
for _ in range(10):
    d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
h2d_gbs = 10 * h.numel() / (time.perf_counter() - t) / 1e9
del h, d

# E-mode (streamed) vs D: FEED, TRANSFER, GENERATE overlapped
sweep = []
n_labels = W * 256
for Ds in (1, 2, 4, 8, 16, 32, 64):
    g = Generator(walkers=W, seed=SEED, epoch_draws=Ds)
    o = torch.empty(W * 8, dtype=torch.int64, device="cuda")
    g.fill(o)  # warm: ring and pinned chunks allocated
    o = torch.empty(n_labels, dtype=torch.int64, device="cuda")
    torch.cuda.synchronize()
    t = time.perf_counter()
    g.fill(o)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t
    sweep.append({"D": Ds, "ns_per_number": dt * 1e9 / n_labels, "G_numbers_per_s": n_labels / dt / 1e9})
    g.close()
    del o
    torch.cuda.empty_cache()

out["fig4_ns_per_number"] = {
    "FEED (host threads, %d cores)" % os.cpu_count(): feed_ns,
    "TRANSFER (24 B at measured pinned H2D %.1f GB/s)" % h2d_gbs: 24 / h2d_gbs,
    "FEED+TRANSFER pipelined (prng_prefetch)": xfer_total_ns,
    "GENERATE (walk kernel, bits resident)": gen_ns,
    "E-mode total (streamed, D=16)": [r for r in sweep if r["D"] == 16][0]["ns_per_number"],
}
out["fig5_sweep"] = sweep
print(json.dumps(out, indent=1))
