"""What bounds C3's FEED pipeline (tool; §V, on-demand bits per round).

    python tools/lr_feed_probe.py "" "GG_FEED_CHUNK_MB=32" "HOST_THREADS=12" ...

Runs C3 (2^24-node list) once to get its per-round active counts, then, for
each config (env assignments, each in its own process), replays the rounds'
windows through prng_epoch_begin / prng_epoch_end (feed threads -> pinned
chunks -> H2D, no kernels) and reports wall ms, the time the feed threads
spent generating (prng_stats.feed_seconds) and the bytes copied: gen-bound
when feed seconds ~ wall, copy-bound when they are well below it.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, os, sys, time
sys.path.insert(0, %(root)r)
import torch
from paper_conf_ipps_banerjeebk12_b200 import Generator
act = json.loads(sys.argv[1])
n = act[0]
g = Generator(walkers=n, seed=0x5EED0003, host_threads=int(os.environ.get("HOST_THREADS", "0")))
g.epoch_reserve(n, 1)
res = []
for rep in range(3):
    s0 = g.stats()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for a in act:
        g.epoch_begin(a, 1)
        g.epoch_end()
    torch.cuda.synchronize()
    wall = time.perf_counter() - t
    s1 = g.stats()
    res.append({"wall_ms": wall * 1e3, "feed_ms": (s1["feed_seconds"] - s0["feed_seconds"]) * 1e3,
                "h2d_gb": (s1["h2d_bytes"] - s0["h2d_bytes"]) / 1e9})
print(json.dumps(res))
"""


def active_counts():
    sys.path.insert(0, ROOT)
    import torch

    import inputs
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    n = 1 << 24
    succ, pred, head = inputs.random_list(n, 0x5EED0003)
    g = Generator(walkers=n, seed=0x5EED0003)
    s, p = torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda()
    rr = torch.empty(n, dtype=torch.int32, device="cuda")
    _, info = g.list_rank(s, p, head, removed_round=rr)
    gone = torch.bincount(rr[rr >= 0].long(), minlength=info["rounds"]).cpu().tolist()
    act = [n]
    for r in range(info["rounds"]):
        act.append(act[-1] - gone[r])
    g.close()
    return act


def main():
    configs = sys.argv[1:] or [""]
    act = active_counts()
    out = {"rounds": len(act), "draws": sum(act), "bits_gb": sum(act) * 24 / 1e9, "runs": {}}
    for c in configs:
        env = dict(os.environ)
        for kv in c.split():
            k, v = kv.split("=")
            env[k] = v
        p = subprocess.run([sys.executable, "-c", CHILD % {"root": ROOT}, json.dumps(act)], env=env,
                           capture_output=True, text=True, timeout=600)
        if p.returncode != 0:
            out["runs"][c or "default"] = {"error": p.stderr[-500:]}
            continue
        r = json.loads(p.stdout.strip().splitlines()[-1])
        best = min(r, key=lambda d: d["wall_ms"])
        best["gbs"] = out["bits_gb"] / (best["wall_ms"] / 1e3)
        out["runs"][c or "default"] = {"best": best, "all": r}
        print(f"[lr-feed] {c or 'default'}: {best['wall_ms']:.1f} ms ({best['gbs']:.1f} GB/s), "
              f"feed threads busy {best['feed_ms']:.1f} ms", file=sys.stderr)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
