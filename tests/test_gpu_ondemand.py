"""On-demand prng_next (header-only device API) vs the oracle, bit-exact.

Epoch rule R10: in an epoch with cursor J0 and depth D, the
i-th prng_next of walker t returns draw J0 + i of walker t; draws a walker
does not use are skipped at epoch end; a walker that sits out an epoch jumps
to the next window.  A draw past the window returns 0 and sets the sticky
overrun flag.
"""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
M32 = 1 << 32


class OracleWalker:
    """Oracle replay of one walker under the epoch rule."""

    def __init__(self, m, seed, t):
        self.m, self.seed, self.t = m, seed, t
        x, y = O.walker_init(m, 64, seed, t)
        self.xy = np.array([x], np.uint64), np.array([y], np.uint64)

    def draw(self, j):
        lib = O.lib()
        x, y = self.xy
        lab = lib.or_walker_draw(self.m, 64, 64, self.seed, self.t, j, x.ctypes.data, y.ctypes.data)
        return int(lab)


def test_uniform_epochs_match_bulk_order():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D, seed = 2048, 5, 21
    g = Generator(walkers=W, seed=seed)
    outs = []
    for e in range(3):
        g.epoch_begin(W, D)
        o = torch.empty(W * D, dtype=torch.int64, device="cuda")
        g.consume(W, uniform=D, out=o)
        g.epoch_end()
        outs.append(o.view(W, D).cpu().numpy().view(np.uint64))
    assert g.check() == 0
    for t in (0, 1, 777, W - 1):
        seq = np.concatenate([o[t] for o in outs])
        assert np.array_equal(seq, O.walker_draws(M32, 64, 64, seed, t, 0, 3 * D))


def test_variable_demand_skips_and_active_subsets():
    # LR-shaped demand: epoch 0 all walkers, varying counts; epoch 1 only
    # walkers [0, 700) active; epoch 2 all again (walkers >= 700 sat out).
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D, seed = 1000, 4, 99
    rng = np.random.default_rng(1)
    g = Generator(walkers=W, seed=seed)
    oracle = {t: OracleWalker(M32, seed, t) for t in (0, 3, 699, 700, 999)}
    J0 = 0
    for e, active in enumerate([W, 700, W]):
        counts = rng.integers(0, D + 1, size=active).astype(np.uint32)
        offs = np.concatenate([[0], np.cumsum(counts)[:-1]]).astype(np.uint64)
        total = int(counts.sum())
        g.epoch_begin(active, D)
        o = torch.zeros(max(total, 1), dtype=torch.int64, device="cuda")
        g.consume(active, counts=torch.from_numpy(counts).cuda(), out=o,
                  offsets=torch.from_numpy(offs.view(np.int64)).cuda())
        g.epoch_end()
        z = o.cpu().numpy().view(np.uint64)
        for t, ow in oracle.items():
            if t >= active:
                continue
            for i in range(int(counts[t])):
                assert int(z[offs[t] + i]) == ow.draw(J0 + i), (e, t, i)
        J0 += D
    assert g.check() == 0


def test_overrun_sets_flag_and_returns_zero():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    from paper_conf_ipps_banerjeebk12_b200._lib import PRNG_E_OVERRUN
    W, D = 256, 2
    g = Generator(walkers=W, seed=4)
    g.epoch_begin(W, D)
    o = torch.empty(W * 3, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=3, out=o)
    g.epoch_end()
    z = o.view(W, 3).cpu().numpy().view(np.uint64)
    assert np.all(z[:, 2] == 0) and np.all(z[:, :2] != 0)
    assert g.check() == PRNG_E_OVERRUN
    assert g.check() == 0  # read-and-clear
    assert np.array_equal(z[5, :2], O.walker_draws(M32, 64, 64, 4, 5, 0, 2))


def test_bulk_after_on_demand_realigns():
    # After an epoch, a bulk fill continues with every walker at draw J0.
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, seed = 512, 8
    g = Generator(walkers=W, seed=seed)
    g.epoch_begin(W, 2)
    g.consume(W, uniform=1, xor_out=torch.empty(W, dtype=torch.int64, device="cuda"))
    g.epoch_end()
    o = torch.empty(W, dtype=torch.int64, device="cuda")
    g.fill(o)
    z = o.cpu().numpy().view(np.uint64)
    for t in (0, 100, W - 1):
        ow = OracleWalker(M32, seed, t)
        ow.draw(0)  # the one used draw; draw 1 skipped
        assert int(z[t]) == ow.draw(2)


def test_epoch_with_walker_list():
    # prng_epoch_begin_list: slot k holds walker ids[k]; numbers per walker are
    # unchanged (draw J0 + i of that walker), only the fed bits differ.
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D, seed = 1000, 3, 17
    g = Generator(walkers=W, seed=seed)
    ids = np.array([999, 3, 500, 0, 42], dtype=np.uint32)
    g.epoch_begin_list(ids, D)
    o = torch.empty(ids.size * D, dtype=torch.int64, device="cuda")
    g.consume(ids.size, uniform=D, out=o)
    g.epoch_end()
    # second epoch over all walkers: listed walkers continue, others start at J0 = 3
    g.epoch_begin(W, 1)
    o2 = torch.empty(W, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=1, out=o2)
    g.epoch_end()
    assert g.check() == 0
    z = o.view(ids.size, D).cpu().numpy().view(np.uint64)
    z2 = o2.cpu().numpy().view(np.uint64)
    for k, t in enumerate(ids):
        assert np.array_equal(z[k], O.walker_draws(M32, 64, 64, seed, int(t), 0, D))
        ow = OracleWalker(M32, seed, int(t))
        for j in range(D):
            ow.draw(j)
        assert int(z2[t]) == ow.draw(3)
    ow = OracleWalker(M32, seed, 7)   # not listed: skipped draws 0..2
    assert int(z2[7]) == ow.draw(3)


def test_epoch_reserve_same_numbers_and_errors():
    """prng_epoch_reserve only pre-allocates: the numbers are unchanged, and
    it is refused inside an open epoch or for empty / oversized windows."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator, PrngError
    W, seed = 4096, 33
    res = []
    for reserve in (False, True):
        g = Generator(walkers=W, seed=seed)
        if reserve:
            g.epoch_reserve(W, 3)
        outs = []
        for A, D in ((W, 3), (W // 2, 2), (W, 1), (100, 3)):
            g.epoch_begin(A, D)
            o = torch.empty(A * D, dtype=torch.int64, device="cuda")
            g.consume(A, uniform=D, out=o)
            g.epoch_end()
            outs.append(o.cpu().numpy())
        res.append(np.concatenate(outs))
        if reserve:
            with pytest.raises(PrngError):
                g.epoch_reserve(0, 1)
            with pytest.raises(PrngError):
                g.epoch_reserve(W + 1, 1)
            g.epoch_begin(10, 1)
            with pytest.raises(PrngError):
                g.epoch_reserve(10, 1)
            g.epoch_end()
        g.close()
    assert np.array_equal(res[0], res[1])


def test_on_demand_bulk_on_demand_keeps_one_sequence():
    """epoch -> ragged bulk fill -> epoch: the second epoch starts at the next
    whole draw after the fill (R10/R11); no draw is emitted twice."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, seed = 300, 23
    g = Generator(walkers=W, seed=seed)
    g.epoch_begin(W, 2)
    a = torch.empty(W * 2, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=2, out=a)
    g.epoch_end()
    n = 3 * W + 5
    b = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(b)
    g.epoch_begin(W, 1)
    c = torch.empty(W, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=1, out=c)
    g.epoch_end()
    a = a.view(W, 2).cpu().numpy().view(np.uint64)
    b = b.cpu().numpy().view(np.uint64)
    c = c.cpu().numpy().view(np.uint64)
    N = 2 * W + n          # bulk positions consumed so far
    J1 = -(-N // W)        # second epoch's first draw
    for t in (0, 4, 5, 150, W - 1):
        ow = OracleWalker(M32, seed, t)
        assert [ow.draw(0), ow.draw(1)] == [int(v) for v in a[t]]
        for j in range(2, 6):
            g_idx = j * W + t - 2 * W
            if g_idx < n:
                assert int(b[g_idx]) == ow.draw(j), (t, j)
        assert int(c[t]) == ow.draw(J1), t
    assert g.check() == 0


def test_full_size_uniform_and_mc_shaped_sampled_parity():
    """The on-demand consumers in bench.py's launch configuration, at full
    size: 2^20 threads x S = 100 prng_next per thread (Fig.4's batch; the
    bench's uniform_S100 line, xor_out and out both checked) and the
    MC-shaped demand (geometric counts, mean 200, cap 600, walker t's draws
    at offsets[t]); sampled walkers against the oracle."""
    import math

    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, S, seed = 1 << 20, 100, 0x5EED0003
    g = Generator(walkers=W, seed=seed)
    g.epoch_begin(W, S)
    o = torch.empty(W * S, dtype=torch.int64, device="cuda")
    xo = torch.empty(W, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=S, out=o)
    g.epoch_end()
    g.epoch_begin(W, S)
    g.consume(W, uniform=S, xor_out=xo)
    g.epoch_end()
    assert g.check() == 0
    z = o.view(W, S)
    x = xo.cpu().numpy().view(np.uint64)
    for t in list(range(0, W, 65521)) + [W - 1]:
        want = O.walker_draws(M32, 64, 64, seed, t, 0, 2 * S)
        assert np.array_equal(z[t].cpu().numpy().view(np.uint64), want[:S]), t
        assert int(x[t]) == int(np.bitwise_xor.reduce(want[S:])), t
    g.close()
    del o, z
    # MC-shaped counts, outputs packed at per-walker offsets
    gen = torch.Generator(device="cpu").manual_seed(7)
    u = torch.rand(W, generator=gen, dtype=torch.float64)
    c = torch.clamp(torch.ceil(torch.log1p(-u) / math.log1p(-1 / 200)), 1, 600).to(torch.int32)
    off = torch.zeros(W, dtype=torch.int64)
    off[1:] = torch.cumsum(c.to(torch.int64), 0)[:-1]
    total = int(c.sum().item())
    g = Generator(walkers=W, seed=seed + 1)
    g.epoch_begin(W, 600)
    o = torch.empty(total, dtype=torch.int64, device="cuda")
    g.consume(W, counts=c.cuda(), out=o, offsets=off.cuda())
    g.epoch_end()
    oc = o.cpu().numpy().view(np.uint64)
    for t in list(range(3, W, 131071)) + [W - 1]:
        n = int(c[t])
        want = O.walker_draws(M32, 64, 64, seed + 1, t, 0, n)
        assert np.array_equal(oc[int(off[t]):int(off[t]) + n], want), t
    g.close()
