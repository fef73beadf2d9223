"""Randomised parity sweep over the generator's parameter space (GPU vs oracle).

Each case draws m (powers of two and others, up to 2^32), l, l0, the variant,
W, the output format, a prefetch depth and a random chunking of the fill
calls, so every kernel path (x2 / x1 TMA, bipartite pair kernel, l = 1 tiles,
generic) meets ragged walker counts and window edges; the bulk sequence must
equal the oracle's (R11) number for number.  Seeded: the same cases every run.
"""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu

MS = [1 << 32, 1 << 31, 1 << 16, 256, 2, 3, 1000, (1 << 30) + 7, (1 << 32) - 5]
LS = [64, 64, 64, 1, 1, 16, 11, 3]
L0S = [64, 64, 0, 1, 63, 7]


def _cases(n=96):
    rng = np.random.default_rng(20121)
    for i in range(n):
        yield dict(m=int(rng.choice(MS)), l=int(rng.choice(LS)), l0=int(rng.choice(L0S)),
                   variant=int(rng.integers(0, 2)), W=int(rng.integers(1, 2600)),
                   draws=int(rng.integers(1, 13)), u32=bool(rng.integers(0, 2)),
                   prefetch=int(rng.integers(0, 3)) * 4, seed=int(rng.integers(0, 2**32)),
                   cuts=int(rng.integers(0, 4)), case=i)


@pytest.mark.parametrize("c", list(_cases()), ids=lambda c: f"case{c['case']}")
def test_random_configuration_parity(c):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    m, W = c["m"], c["W"]
    g = Generator(walkers=W, seed=c["seed"], m=m, walk_len=c["l"], burnin_len=c["l0"],
                  variant=c["variant"], epoch_draws=int(1 + c["case"] % 5))
    if c["prefetch"]:
        g.prefetch(c["prefetch"])
    n = W * c["draws"] + (c["case"] % 7)
    want = O.bulk_v(m, c["l"], c["l0"], c["variant"], c["seed"], W, 0, n)
    words_per = 1 if m <= (1 << 16) else 2
    if c["u32"]:
        out = torch.empty(n * words_per, dtype=torch.int32, device="cuda")
        unit = words_per
    else:
        out = torch.empty(n, dtype=torch.int64, device="cuda")
        unit = 1
    rng = np.random.default_rng(c["case"])
    cuts = sorted(set(int(v) for v in rng.integers(1, n, c["cuts"]))) if n > 1 else []
    lo = 0
    for hi in cuts + [n]:
        g.fill(out[lo * unit:hi * unit])
        lo = hi
    torch.cuda.synchronize()
    if c["u32"] and words_per == 1:
        got = out.cpu().numpy().view(np.uint32).astype(np.uint64)
    else:
        got = out.cpu().numpy().view(np.uint64)
    assert np.array_equal(got, want), c
    assert g.check() == 0
    g.close()
