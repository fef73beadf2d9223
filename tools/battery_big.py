"""Crush-scale battery on GPU output (tool; §IV-B,
Table III: SmallCrush 15/15, Crush 14/15, BigCrush 13/15).

    python tools/battery_big.py [--log2-words 33] [--streams 0,1] > profiles/r02_battery.json

Streams 2^log2-words u32 words (default 2^33 = 2^32 labels) of the generator
through the 15 streaming statistics of tests/battery_gpu.py (computed with
torch on the GPU; test infrastructure, not the product path):
  bulk          C2 generator (m = 2^32, l = l0 = 64, 2^20 walkers), bulk order
  walker-major  the same walk with 4096 walkers, each fill of 2^28 labels
                transposed so every walker's 2^16 consecutive draws are adjacent
and, as negative controls on 2^28 words: l = 1 and l = 16 (walker-major) and
the 32-bit LCG of Numerical Recipes (a = 1664525, c = 1013904223).
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import battery_gpu as G  # noqa: E402
from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

CHUNK = 1 << 28   # labels per fill (2 GiB)
SUB = 1 << 26     # labels per feed() call


def gen_chunks(total_labels, walkers, walk_len=64, seed=0x5EED00B1, walker_major=False,
               variant=0, bit_source=0):
    # few walkers: deep ring slots, so each streamed window is ~100 MB of bits
    g = Generator(walkers=walkers, seed=seed, walk_len=walk_len,
                  epoch_draws=16 if walkers >= (1 << 18) else 1024, variant=variant,
                  bit_source=bit_source)
    out = torch.empty(min(CHUNK, total_labels), dtype=torch.int64, device="cuda")
    done = 0
    while done < total_labels:
        n = min(CHUNK, total_labels - done)
        o = out[:n]
        g.fill(o)
        if walker_major:
            o = o.view(n // walkers, walkers).t().contiguous().view(-1)
        yield o
        done += n
    g.close()


def lcg_chunks(total_labels):
    """Numerical Recipes' 32-bit LCG, label i = words 2i (low), 2i+1 (high)."""
    a, c, M = 1664525, 1013904223, 0xFFFFFFFF
    blk = 1 << 12
    x = np.empty(blk, dtype=np.uint64)
    s = 12345
    for i in range(blk):
        s = (a * s + c) & M
        x[i] = s
    A, C = 1, 0  # x[i + blk] = A x[i] + C
    for _ in range(blk):
        A, C = (a * A) & M, (a * C + c) & M
    A, C = np.uint64(A), np.uint64(C)
    words = 2 * total_labels
    out = np.empty(words, dtype=np.uint64)
    out[:blk] = x
    for j in range(blk, words, blk):
        out[j:j + blk] = (A * out[j - blk:j] + C) & np.uint64(M)
    lab = (out[0::2] | (out[1::2] << np.uint64(32))).view(np.int64)
    for i in range(0, total_labels, CHUNK):
        yield torch.from_numpy(lab[i:i + CHUNK]).cuda()


def run_stream(chunks, tests):
    secs = {t.name: 0.0 for t in tests}
    labels = 0
    t_gen = 0.0
    t0 = time.perf_counter()
    for ch in chunks:
        torch.cuda.synchronize()
        t_gen += time.perf_counter() - t0
        for i in range(0, ch.numel(), SUB):
            sub = ch[i:i + SUB]
            for t in tests:
                a = time.perf_counter()
                t.feed(sub)
                torch.cuda.synchronize()
                secs[t.name] += time.perf_counter() - a
        labels += ch.numel()
        t0 = time.perf_counter()
    res = {}
    for t in tests:
        a = time.perf_counter()
        p = t.pvalue()
        secs[t.name] += time.perf_counter() - a
        res[t.name] = {"p": float(f"{p:.4g}"), "verdict": G.verdict(t, p),
                       "seconds": round(secs[t.name], 2)}
    passed = sum(1 for v in res.values() if v["verdict"] == "pass")
    return {"words": 2 * labels, "labels": labels, "passed": f"{passed}/{len(tests)}",
            "failed": sorted(k for k, v in res.items() if v["verdict"] == "fail"),
            "generate_seconds": round(t_gen, 2), "tests": res}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--log2-words", type=int, default=33)
    ap.add_argument("--log2-words-controls", type=int, default=28)
    ap.add_argument("--streams", default="", help="comma-separated stream indices (default: 0-4)")
    ap.add_argument("--log2-words-extra", type=int, default=33,
                    help="size of streams 5 (bipartite walk) and 6 (glibc rand_r seed bits)")
    args = ap.parse_args()
    L = 1 << (args.log2_words - 1)
    Lx = 1 << (args.log2_words_extra - 1)
    Lc = 1 << (args.log2_words_controls - 1)
    rep = {"what": "15 streaming Crush-style statistics (tests/battery_gpu.py) computed with torch "
                   "on the GPU; fail = one-sided p outside [1e-4, 1-1e-4] or two-sided p < 1e-4",
           "paper": "Table III (TestU01): SmallCrush 15/15, Crush 14/15, BigCrush 13/15",
           "notes": "matrix_rank_300 reads the first 2^15 matrices (4.9e7 labels) of each stream; "
                    "every other statistic reads the whole stream",
           "streams": {}}
    runs = [
        ("bulk l=64", lambda: gen_chunks(L, 1 << 20)),
        ("walker-major l=64", lambda: gen_chunks(L, 4096, walker_major=True)),
        ("control: bulk l=1", lambda: gen_chunks(Lc, 1 << 20, walk_len=1)),
        ("control: walker-major l=16", lambda: gen_chunks(Lc, 4096, walk_len=16, walker_major=True)),
        ("control: 32-bit LCG", lambda: lcg_chunks(Lc)),
        # f1: the bipartite sigma / sigma^-1 walk; f3: the paper's glibc rand_r
        # LCG as the seed-bit source (§III-B), both C2-shaped, bulk order
        ("bipartite l=64", lambda: gen_chunks(Lx, 1 << 20, variant=1)),
        ("rand_r seed bits l=64", lambda: gen_chunks(Lx, 1 << 20, bit_source=1)),
    ]
    runs = [runs[int(i)] for i in args.streams.split(",")] if args.streams else runs[:5]
    for name, mk in runs:
        t = time.perf_counter()
        r = run_stream(mk(), G.crush_scale_tests())
        r["seconds"] = round(time.perf_counter() - t, 1)
        rep["streams"][name] = r
        print(f"[battery] {name}: {r['passed']} in {r['seconds']} s, failed {r['failed']}",
              file=sys.stderr)
        torch.cuda.empty_cache()
    print(json.dumps(rep, indent=1))


if __name__ == "__main__":
    main()
