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


def _od_cases(n=24):
    rng = np.random.default_rng(77)
    for i in range(n):
        ops = [str(rng.choice(["epoch", "list", "bulk"])) for _ in range(5)]
        yield dict(m=int(rng.choice([1 << 32, 256, 1000, (1 << 32) - 5])),
                   l=int(rng.choice([64, 64, 1, 16])), variant=int(rng.integers(0, 2)),
                   W=int(rng.integers(2, 1500)), seed=int(rng.integers(0, 2**32)), ops=ops, case=i)


class _Replay:
    """Oracle replay of every walker under the epoch rule R10: a walker's next
    number walks the bits of the draw it is given from the vertex it is at
    (draws it skipped are never walked), so numbers after skipped draws are
    NOT the bulk table's."""

    def __init__(self, m, l, variant, seed, W):
        self.m, self.l, self.v, self.seed = m, l, variant, seed
        self.x = np.zeros(W, np.uint64)
        self.y = np.zeros(W, np.uint64)
        for t in range(W):
            O.lib().or_walker_init_v(m, 64, variant, seed, t, self.x[t:].ctypes.data,
                                     self.y[t:].ctypes.data)

    def draw(self, t, j):
        return int(O.lib().or_walker_draw_v(self.m, self.l, 64, self.v, self.seed, t, j,
                                            self.x[t:].ctypes.data, self.y[t:].ctypes.data))


@pytest.mark.parametrize("c", list(_od_cases()), ids=lambda c: f"od{c['case']}")
def test_random_on_demand_sequences(c):
    """Random sequences of on-demand epochs (walker prefixes with random
    per-thread counts, explicit walker lists) and bulk fills: every number is
    the draw the epoch rule R10 and the bulk order R11 assign, replayed walker
    by walker on the oracle."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, m, l, v, seed = c["W"], c["m"], c["l"], c["variant"], c["seed"]
    rng = np.random.default_rng(1000 + c["case"])
    ref = _Replay(m, l, v, seed, W)
    g = Generator(walkers=W, seed=seed, m=m, walk_len=l, variant=v)
    N, J0 = 0, None  # bulk position; epoch cursor (None: not started -> next whole draw)
    for op in c["ops"]:
        if op == "bulk":
            n = int(rng.integers(1, 2 * W))
            o = torch.empty(n, dtype=torch.int64, device="cuda")
            g.fill(o)
            want = [ref.draw(pos % W, pos // W) for pos in range(N, N + n)]
            assert [int(z) for z in o.cpu().numpy().view(np.uint64)] == want, (c, op)
            N += n
            J0 = None
            continue
        start = J0 if J0 is not None else -(-N // W)
        D = int(rng.integers(1, 5))
        A = int(rng.integers(1, W + 1))
        if op == "epoch":
            walkers = np.arange(A)
            g.epoch_begin(A, D)
        else:
            walkers = rng.permutation(W)[:A].astype(np.uint32)
            g.epoch_begin_list(walkers, D)
        cnt = rng.integers(0, D + 1, A).astype(np.int32)
        off = np.zeros(A, np.int64)
        off[1:] = np.cumsum(cnt)[:-1]
        o = torch.empty(max(1, int(cnt.sum())), dtype=torch.int64, device="cuda")
        g.consume(A, counts=torch.from_numpy(cnt).cuda(), out=o, offsets=torch.from_numpy(off).cuda())
        g.epoch_end()
        got = o.cpu().numpy().view(np.uint64)
        for k in range(A):
            t = int(walkers[k])
            want = [ref.draw(t, start + i) for i in range(int(cnt[k]))]
            assert [int(z) for z in got[off[k]:off[k] + cnt[k]]] == want, (c, op, k)
        J0 = start + D
        N = J0 * W
    assert g.check() == 0
    g.close()
