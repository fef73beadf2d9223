"""Python quickstart (needs a GPU): the generator's public API in one page.

    python examples/quickstart.py

1. bulk numbers (prng_fill, Alg.2) into a CUDA tensor, as 64-bit labels
   and as 32-bit words;
2. the same with the seed bits made resident first (prng_prefetch) and with
   the numbers landing in host memory (prng_fill_host);
3. on-demand numbers inside a kernel (prng_next via an epoch; here the
   library's own consumer kernel gg_consume with a different count per thread);
4. the paper's two applications: list ranking (Alg.3) and Monte Carlo photon
   migration (Alg.4);
5. other seed-bit sources: glibc rand_r, and the generator itself on the host.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import inputs  # noqa: E402
from paper_conf_ipps_banerjeebk12_b200 import (PRNG_BITS_GGCPU, PRNG_BITS_RANDR,  # noqa: E402
                                               Generator)


def main():
    W = 1 << 16                                    # walkers (one stream each)
    g = Generator(walkers=W, seed=2012)            # Alg.1: start + 64-step burn-in
    labels = torch.empty(W * 4, dtype=torch.int64, device="cuda")
    g.fill(labels)                                 # next W*4 numbers, order g = j*W + t
    words = torch.empty(W * 2, dtype=torch.int32, device="cuda")
    g.fill(words)                                  # 2 words per 64-bit label (m = 2^32)
    print("bulk:", [hex(v) for v in labels[:3].cpu().numpy().view(np.uint64)])

    g.prefetch(8)                                  # bits of the next 8 draws resident in HBM
    g.fill(labels)                                 # kernels only (K-mode)
    host = np.empty(W, dtype=np.uint64)
    g.fill_host(host)                              # host buffer; H2D/D2H overlapped
    print("fill_host:", hex(int(host[0])), "tell:", g.tell())

    counts = torch.randint(0, 5, (W,), dtype=torch.int32, device="cuda")
    offsets = torch.zeros(W, dtype=torch.int64, device="cuda")
    offsets[1:] = torch.cumsum(counts.to(torch.int64), 0)[:-1]
    out = torch.empty(int(counts.sum()), dtype=torch.int64, device="cuda")
    with g.epoch(W, 4):                            # draws J0..J0+3 of every walker resident
        g.consume(W, counts=counts, out=out, offsets=offsets)  # thread t: counts[t] x prng_next
    print("on demand:", out.numel(), "numbers, overrun flag", g.check())
    g.close()

    n = 1 << 20
    succ, pred, head = inputs.random_list(n, 7)
    lr = Generator(walkers=n, seed=3)
    rank, info = lr.list_rank(torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda(), head)
    print("list ranking:", info["rounds"], "rounds,", info["draws"], "draws, tail rank",
          int(rank.max()))
    lr.close()

    layers = ((1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2))
    mc = Generator(walkers=1 << 14, seed=4)
    r = mc.mc_run(layers, photons_total=1 << 16)
    print("Monte Carlo: R_d = %.4f, T_t = %.4f" % (r["R_d"] / r["launched"], r["T_t"] / r["launched"]))
    mc.close()

    for src, name in ((PRNG_BITS_RANDR, "glibc rand_r"), (PRNG_BITS_GGCPU, "host generator")):
        h = Generator(walkers=1024, seed=5, bit_source=src)
        o = torch.empty(1024, dtype=torch.int64, device="cuda")
        h.fill(o)
        print(name, "bits:", hex(int(o[0].cpu().numpy().view(np.uint64))))
        h.close()


if __name__ == "__main__":
    main()
