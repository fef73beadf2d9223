"""Interleaved A/B of host FEED settings (tool; §IV-A Fig.4-5).

    python tools/feed_ab.py [--reps 3] "" "GG_FEED_RATE=0" "GG_FEED_RATE=70" ...

Host-side rates on the GPU box drift between runs by 10-30%, so configs are
run round-robin (A B C A B C ...), each in a fresh process, and medians are
reported.  Each process measures, for its env settings:
  e2e   -- prng_fill_host of 2^20 walkers x 512 draws (the bench's C2 e2e
           step: 12.9 GB of seed bits, labels to pinned host memory; AB_E2E_DRAWS
           changes the draws), best wall time of 2;
  lr    -- C3's FEED pipeline: C3's per-round active counts (computed once
           by the parent) replayed through prng_epoch_begin / prng_epoch_end
           (bits generated and copied, no kernels), wall time;
  c3    -- the full C3 list ranking (median of 3 after one untimed call).
HOST_THREADS=n sets the pool size (host_threads); the library's other
knobs are read from the environment.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import json, os, sys, time
sys.path.insert(0, %(root)r)
import torch
from paper_conf_ipps_banerjeebk12_b200 import Generator
act = json.load(open(sys.argv[1]))
ht = int(os.environ.get("HOST_THREADS", "0"))
W = 1 << 20
g = Generator(walkers=W, seed=0x5EED0002, epoch_draws=16, host_threads=ht)
D = int(os.environ.get("AB_E2E_DRAWS", "512"))  # 512: the bench e2e step (2^29 labels)
host = torch.empty(W * D, dtype=torch.int64).pin_memory()
g.fill_host(host, n=W * 8)
g.mark()
e2e = []
for _ in range(2):
    g.rewind()
    torch.cuda.synchronize()
    t = time.perf_counter()
    g.fill_host(host)
    torch.cuda.synchronize()
    e2e.append(time.perf_counter() - t)
writers = g.stats()["feed_pace_mbs"]
g.close()
n = act[0]
g = Generator(walkers=n, seed=0x5EED0003, host_threads=ht)
g.epoch_reserve(n, 1)
lr = []
for _ in range(3):
    torch.cuda.synchronize()
    t = time.perf_counter()
    for a in act:
        g.epoch_begin(a, 1)
        g.epoch_end()
    torch.cuda.synchronize()
    lr.append(time.perf_counter() - t)
g.close()
# the full C3 list ranking (kernels + on-demand FEED), median of 3 after one untimed call
import inputs
succ, pred, head = inputs.random_list(n, 0x5EED0003)
g = Generator(walkers=n, seed=0x5EED0003, host_threads=ht)
s_t, p_t = torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda()
g.list_rank(s_t, p_t, head)
c3 = []
for _ in range(3):
    torch.cuda.synchronize()
    t = time.perf_counter()
    g.list_rank(s_t, p_t, head)
    torch.cuda.synchronize()
    c3.append(time.perf_counter() - t)
g.close()
print(json.dumps({"c3_ms": sorted(c3)[1] * 1e3, "e2e_gnum_s": W * D / min(e2e) / 1e9, "lr_ms": min(lr) * 1e3, "pace_mbs": writers}))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("configs", nargs="*")
    args = ap.parse_args()
    configs = args.configs or [""]
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from lr_feed_probe import active_counts
    act = active_counts()
    path = os.path.join(ROOT, "gpurun_out", "feed_ab_act.json")
    os.makedirs(os.path.dirname(path), exist_ok=True)
    with open(path, "w") as f:
        json.dump(act, f)
    runs = {c or "default": [] for c in configs}
    for rep in range(args.reps):
        for c in configs:
            env = dict(os.environ)
            for kv in c.split():
                k, v = kv.split("=")
                env[k] = v
            p = subprocess.run([sys.executable, "-c", CHILD % {"root": ROOT}, path], env=env,
                               capture_output=True, text=True, timeout=600)
            r = (json.loads(p.stdout.strip().splitlines()[-1]) if p.returncode == 0
                 else {"error": p.stderr[-300:]})
            runs[c or "default"].append(r)
            print(f"[feed-ab] rep {rep} {c or 'default'}: {r}", file=sys.stderr)
    out = {"lr_bits_gb": sum(act) * 24 / 1e9, "configs": {}}
    for c, rs in runs.items():
        ok = [r for r in rs if "error" not in r]
        if not ok:
            out["configs"][c] = {"error": rs[-1]}
            continue
        out["configs"][c] = {
            "e2e_gnum_s_median": statistics.median(r["e2e_gnum_s"] for r in ok),
            "lr_ms_median": statistics.median(r["lr_ms"] for r in ok),
            "c3_ms_median": statistics.median(r["c3_ms"] for r in ok),
            "pace_mbs": ok[0]["pace_mbs"], "runs": ok}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
