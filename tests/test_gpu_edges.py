"""Edge cases of the CUDA path vs the oracle (bit-exact): degenerate and
ragged sizes, the largest walker counts, the top of the walker-id space.

Readings: R9 (walker ids < 2^24 per seed, counter layout), R11 (bulk order
g = j*W + t, fills continue from the running N), R12 (u32 words).
"""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
M32 = 1 << 32


def G(**kw):
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    return Generator(**kw)


def u64(t):
    return t.cpu().numpy().view(np.uint64)


@pytest.mark.parametrize("W", [1, 2, 31, 33, 63, 65, 1000])
def test_ragged_walker_counts_and_fill_sizes(W):
    """Warps with idle lanes (W not a multiple of 32/64) and fills that stop
    mid-draw: the concatenation equals the oracle's bulk sequence."""
    import torch
    seed = 0x5EED00E0 + W
    sizes = [1, W + 3, 5 * W - 1, 7, 2 * W]
    total = sum(sizes)
    want = O.bulk(M32, 64, 64, seed, W, 0, total)
    g = G(walkers=W, seed=seed, epoch_draws=2)
    got = []
    for n in sizes:
        o = torch.empty(n, dtype=torch.int64, device="cuda")
        g.fill(o)
        got.append(u64(o))
    assert np.array_equal(np.concatenate(got), want)
    assert g.tell() == total


def test_zero_length_fill_is_a_no_op():
    import torch
    g = G(walkers=64, seed=3)
    o = torch.empty(0, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert g.tell() == 0
    o = torch.empty(64, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert np.array_equal(u64(o), O.bulk(M32, 64, 64, 3, 64, 0, 64))


def test_top_of_walker_id_space():
    """walker_base + walkers = 2^24 is the largest legal shard (R9); one more
    walker is refused at create time."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    W, base, seed = 96, (1 << 24) - 96, 77
    g = G(walkers=W, seed=seed, walker_base=base)
    o = torch.empty(3 * W, dtype=torch.int64, device="cuda")
    g.fill(o)
    z = u64(o).reshape(3, W)
    for t in (0, 1, 50, W - 1):
        assert np.array_equal(z[:, t], O.walker_draws(M32, 64, 64, seed, base + t, 0, 3))
    g.close()
    with pytest.raises(PrngError):
        G(walkers=W, seed=seed, walker_base=base + 1)


def test_max_walkers_sampled_parity():
    """2^24 walkers (the per-seed maximum): two draws each, sampled walkers."""
    import torch
    W, seed = 1 << 24, 0x5EED00E1
    g = G(walkers=W, seed=seed)
    o = torch.empty(2 * W, dtype=torch.int64, device="cuda")
    g.fill(o)
    z = u64(o).reshape(2, W)
    for t in list(range(0, W, 1 << 20)) + [W - 1, W - 33]:
        assert np.array_equal(z[:, t], O.walker_draws(M32, 64, 64, seed, t, 0, 2)), t


def test_u32_words_ragged_and_small_m():
    """R12: m = 2^32 -> 2 words per label (even counts only); m <= 2^16 -> 1."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    g = G(walkers=40, seed=9)
    o = torch.empty(2 * 45, dtype=torch.int32, device="cuda")
    g.fill(o)
    assert np.array_equal(o.cpu().numpy().view(np.uint64), O.bulk(M32, 64, 64, 9, 40, 0, 45))
    with pytest.raises(PrngError):
        g.fill(torch.empty(3, dtype=torch.int32, device="cuda"))
    g2 = G(walkers=40, seed=9, m=1 << 16)
    o = torch.empty(45, dtype=torch.int32, device="cuda")
    g2.fill(o)
    want = O.bulk(1 << 16, 64, 64, 9, 40, 0, 45)
    assert np.array_equal(o.cpu().numpy().view(np.uint32).astype(np.uint64), want)


def test_misaligned_output_is_refused_without_side_effects():
    """Labels are stored whole: a u32 buffer for m = 2^32 must be 8-B aligned."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    g = G(walkers=64, seed=5)
    buf = torch.empty(2 * 64 + 1, dtype=torch.int32, device="cuda")
    with pytest.raises(PrngError):
        g.fill(buf[1:], n=2 * 64)
    assert g.tell() == 0
    g.fill(buf[:-1])  # still usable, sequence unchanged
    assert np.array_equal(buf[:-1].cpu().numpy().view(np.uint64), O.bulk(M32, 64, 64, 5, 64, 0, 64))
    g2 = G(walkers=64, seed=5, m=1 << 16)  # one word per label: 4-B alignment is enough
    g2.fill(buf[1:], n=64)
    want = O.bulk(1 << 16, 64, 64, 5, 64, 0, 64)
    assert np.array_equal(buf[1:65].cpu().numpy().view(np.uint32).astype(np.uint64), want)


def test_smallest_modulus():
    """m = 2: a 4-vertex graph; still the oracle's sequence."""
    import torch
    g = G(walkers=70, seed=4, m=2)
    o = torch.empty(70 * 9, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert np.array_equal(u64(o), O.bulk(2, 64, 64, 4, 70, 0, 70 * 9))


def test_on_demand_single_walker_single_draw():
    import torch
    g = G(walkers=1, seed=12)
    g.epoch_begin(1, 1)
    o = torch.empty(1, dtype=torch.int64, device="cuda")
    g.consume(1, uniform=1, out=o)
    g.epoch_end()
    assert int(u64(o)[0]) == int(O.walker_draws(M32, 64, 64, 12, 0, 0, 1)[0])
    assert g.check() == 0


def test_binding_rejects_unsafe_outputs():
    """The Python binding checks what the C ABI cannot: the output tensor is
    contiguous, holds n numbers and lives on the handle's device (host memory
    for fill_host); nothing is generated on a refusal."""
    import torch
    g = G(walkers=64, seed=1)
    d = torch.empty(256, dtype=torch.int64, device="cuda")
    for bad in (lambda: g.fill(d[::2]),                         # strided view
                lambda: g.fill(d, n=257),                       # n > numel
                lambda: g.fill(torch.empty(8, dtype=torch.int64)),  # host tensor
                lambda: g.fill_host(d),                         # device tensor
                lambda: g.fill_host(torch.empty(8, dtype=torch.int64), n=9),
                lambda: g.fill_host(np.empty((4, 4), dtype=np.uint64)[:, ::2])):
        with pytest.raises(ValueError):
            bad()
    assert g.tell() == 0
    g.fill(d, n=100)
    assert g.tell() == 100
    g.close()
