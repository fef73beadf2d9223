"""Fig.3 analogue on B200 (tool; §IV-A Fig.3: time to generate N
random numbers, N = 5 M ... 1000 M, the paper's hybrid at ~0.07 GNumbers/s).

    python tools/fig3.py > profiles/r02_fig3.json

C2 generator (m = 2^32, l = l0 = 64), 2^20 walkers, 64-bit numbers to device
memory, for N in the paper's range.  Per N, three numbers (best of 3, after a
warm-up call of the same size):
  create_ms  -- prng_create: Alg.1 for 2^20 walkers (host feed of the start
                and burn-in bits, H2D, init kernel);
  k_gnum_s   -- K-mode: prng_fill with the N numbers' seed bits already in HBM
                (prng_prefetch, untimed), device-timed with CUDA events;
  e_gnum_s   -- E-mode: prng_fill with the host FEED streaming the bits during
                the walk (the paper's hybrid), wall time to the last number.
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


def main():
    rows = []
    out = torch.empty(1000 * 1000 * 1000, dtype=torch.int64, device="cuda")
    for n_m in (5, 10, 50, 100, 500, 1000):
        n = n_m * 1000 * 1000
        draws = -(-n // W)
        o = out[:n]
        creates, ks, es = [], [], []
        for rep in range(4):
            torch.cuda.synchronize()
            t = time.perf_counter()
            g = Generator(walkers=W, seed=SEED)
            torch.cuda.synchronize()
            creates.append(time.perf_counter() - t)
            # E-mode: bits streamed by the host feed during the walk
            torch.cuda.synchronize()
            t = time.perf_counter()
            g.fill(o)
            torch.cuda.synchronize()
            es.append(time.perf_counter() - t)
            # K-mode: the same numbers again with their bits resident
            g.close()
            g = Generator(walkers=W, seed=SEED)
            g.prefetch(draws)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            g.fill(o)
            e1.record()
            torch.cuda.synchronize()
            ks.append(e0.elapsed_time(e1) / 1e3)
            g.close()
        # rep 0 is the warm-up (allocations, first feed-thread start)
        creates, ks, es = creates[1:], ks[1:], es[1:]
        rows.append({"N": n, "draws_per_walker": draws,
                     "create_ms": round(min(creates) * 1e3, 2),
                     "k_gnum_s": round(n / min(ks) / 1e9, 2),
                     "e_gnum_s": round(n / min(es) / 1e9, 3),
                     "e_ms": round(min(es) * 1e3, 1), "k_ms": round(min(ks) * 1e3, 3)})
        print(json.dumps(rows[-1]), file=sys.stderr)
        torch.cuda.empty_cache()
    print(json.dumps({"config": "m=2^32, l=l0=64, 2^20 walkers, 64-bit numbers to device memory",
                      "paper": "Fig.3: hybrid CPU+GPU ~0.07 GNumbers/s on a Tesla C1060 + Core i7-980",
                      "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
