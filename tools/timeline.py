"""Fig.4 timeline analogue (tool; §IV-A Fig.4: FEED / TRANSFER /
GENERATE overlap, "the GPU is idle for about 20%").

    python tools/timeline.py > profiles/r02_timeline.json

Runs the C2 generator (m = 2^32, l = l0 = 64, 2^20 walkers) in E-mode (seed
bits streamed by the host FEED during the walk) with the library's timeline
recorder on (GG_TIMELINE, prng_capi.cu): every FEED chunk (host feed threads),
H2D copy, walk kernel and D2H copy as an interval on one clock.  For each
run it reports, over the span of the run: the busy fraction of each resource
(union of its intervals), the GPU idle fraction (no walk kernel running), and
how much of the time FEED, TRANSFER and GENERATE ran concurrently.
"""
import json
import os
import sys
import tempfile
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def length(iv):
    return sum(b - a for a, b in iv)


def intersect(x, y):
    i = j = 0
    out = []
    while i < len(x) and j < len(y):
        a, b = max(x[i][0], y[j][0]), min(x[i][1], y[j][1])
        if a < b:
            out.append([a, b])
        if x[i][1] < y[j][1]:
            i += 1
        else:
            j += 1
    return out


def analyse(rows, t_lo=None, t_hi=None):
    kinds = {}
    for k, a, b in rows:
        kinds.setdefault(k, []).append([a, b])
    lo = min(a for _, a, _ in rows) if t_lo is None else t_lo
    hi = max(b for _, _, b in rows) if t_hi is None else t_hi
    span = hi - lo
    u = {k: union(v) for k, v in kinds.items()}
    res = {"span_ms": span / 1e3, "intervals": {k: len(v) for k, v in kinds.items()},
           "busy_frac": {k: length(v) / span for k, v in u.items()}}
    if "walk" in u:
        res["gpu_idle_frac"] = 1.0 - length(u["walk"]) / span
    if "feed" in u and "h2d" in u:
        fh = intersect(u["feed"], u["h2d"])
        res["feed_and_h2d_frac"] = length(fh) / span
        if "walk" in u:
            res["feed_h2d_walk_frac"] = length(intersect(fh, u["walk"])) / span
    return res


def run(kind, W=1 << 20, draws=512, D=16):
    import torch

    from paper_conf_ipps_banerjeebk12_b200 import Generator
    path = tempfile.mktemp(suffix=".json")
    os.environ["GG_TIMELINE"] = path
    g = Generator(walkers=W, seed=0x5EED0002, epoch_draws=D)
    del os.environ["GG_TIMELINE"]
    n = W * draws
    if kind == "fill":
        out = torch.empty(n, dtype=torch.int64, device="cuda")
        g.fill(out[:W * D])  # warm: allocations, feed threads
        torch.cuda.synchronize()
        t = time.perf_counter()
        g.fill(out[W * D:])
        torch.cuda.synchronize()
    else:
        out = torch.empty(n, dtype=torch.int64).pin_memory()
        g.fill_host(out[:W * D])
        t = time.perf_counter()
        g.fill_host(out[W * D:])
    wall = time.perf_counter() - t
    g.close()
    with open(path) as f:
        rows = json.load(f)
    os.unlink(path)
    # the warm-up call (one ring slot, one walk kernel) completed before the
    # timed call started: keep the intervals that start after its walk ended
    warm_end = min(b for k, a, b in rows if k == "walk")
    timed = [r for r in rows if r[1] >= warm_end]
    res = analyse(timed)
    res.update({"call": "prng_fill (device output)" if kind == "fill" else
                "prng_fill_host (host output, D2H overlapped)",
                "numbers": n - W * D, "wall_ms": wall * 1e3,
                "numbers_per_s": (n - W * D) / wall, "epoch_draws": D})
    return res


def main():
    out = {"config": "C2 generator, m=2^32, l=l0=64, 2^20 walkers, E-mode (bits streamed by "
                     "the host FEED during the walk), ring slots of D=16 draws",
           "what": "busy_frac = union of each resource's intervals / span of the timed call; "
                   "gpu_idle_frac = share of the span with no walk kernel running "
                   "(the paper's Fig.4 observation: 'the GPU is idle for about 20%')",
           "runs": [run("fill"), run("fill_host")]}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
