"""C3 list-ranking timeline (tool; §V, on-demand bits per round).

    python tools/lr_timeline.py > gpurun_out/lr_timeline.json

Runs gg_list_rank on the 2^24-node list twice on one handle with the
library's timeline recorder on (GG_TIMELINE): FEED chunks, H2D copies, the
host waiting for a free pinned chunk ("ring_wait"), and per round the host
time in prng_epoch_begin ("lr.begin"), in the next round's prefeed
("lr.prefeed"), waiting for the survivor count ("lr.wait") and the round's
kernels on the device ("lr.kernels").  For the second (timed) call it reports
each resource's busy fraction, the H2D idle gaps (> 20 us) with what the host
and the GPU were doing during each, and the copy rate while busy.
"""
import json
import os
import sys
import tempfile
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from timeline import intersect, length, union  # noqa: E402


def main():
    import torch

    import inputs
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    n = 1 << 24
    succ, pred, head = inputs.random_list(n, 0x5EED0003)
    s, p = torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda()
    path = tempfile.mktemp(suffix=".json")
    os.environ["GG_TIMELINE"] = path
    g = Generator(walkers=n, seed=0x5EED0003)
    del os.environ["GG_TIMELINE"]
    walls = []
    for rep in range(2):
        torch.cuda.synchronize()
        time.sleep(0.05)
        t = time.perf_counter()
        _, info = g.list_rank(s, p, head)
        torch.cuda.synchronize()
        walls.append((time.perf_counter() - t) * 1e3)
    h2d_bytes = g.stats()["h2d_bytes"]
    g.close()
    with open(path) as f:
        rows = json.load(f)
    os.unlink(path)
    # split the two calls at the largest gap between consecutive interval starts
    rows.sort(key=lambda r: r[1])
    gaps = [(rows[i + 1][1] - rows[i][2], i) for i in range(len(rows) - 1)]
    cut = max(gaps)[1] + 1
    timed = rows[cut:]
    lo = min(a for _, a, _ in timed)
    hi = max(b for _, _, b in timed)
    kinds = {}
    for k, a, b in timed:
        kinds.setdefault(k, []).append([a, b])
    u = {k: union(v) for k, v in kinds.items()}
    span = hi - lo
    res = {"wall_ms": walls, "info": info, "span_ms": span / 1e3,
           "busy_frac": {k: length(v) / span for k, v in u.items()},
           "intervals": {k: len(v) for k, v in kinds.items()}}
    h2d = u.get("h2d", [])
    # idle gaps of the copy stream inside the span (incl. before the first copy)
    edges = [[lo, lo]] + h2d + [[hi, hi]]
    idle = []
    for x, y in zip(edges, edges[1:]):
        a, b = x[1], y[0]
        if b - a > 20.0:
            during = {k: round(length(intersect([[a, b]], v)) / (b - a), 3)
                      for k, v in u.items() if k != "h2d" and intersect([[a, b]], v)}
            idle.append({"at_ms": round((a - lo) / 1e3, 3), "us": round(b - a, 1), "during": during})
    res["h2d_idle_gaps"] = idle
    res["h2d_idle_ms"] = sum(g_["us"] for g_ in idle) / 1e3
    res["h2d_busy_ms"] = length(h2d) / 1e3
    res["h2d_gb_both_calls"] = h2d_bytes / 1e9
    # per-round picture: begin / prefeed / wait host spans and the kernels
    res["rounds"] = [[k, round((a - lo) / 1e3, 3), round((b - a) / 1e3, 3)]
                     for k, a, b in timed if k.startswith("lr.")]
    res["raw_ms"] = [[k, round((a - lo) / 1e3, 4), round((b - lo) / 1e3, 4)] for k, a, b in timed]
    print(json.dumps(res))


if __name__ == "__main__":
    main()
