"""SmallCrush-style battery (tests/battery.py) on the oracle's output, with
the battery's own power pinned on known-bad inputs.

The paper reports that the GG generator passes DIEHARD and TestU01 (P:18
§IV-B, Tables II-III).  Here the battery runs on C2-type output of the
oracle (m = 2^32, l = l0 = 64) in two orders: bulk order g = j*W + t (R11)
and walker-major order (each walker's consecutive draws, where the walk
could leave correlations).  It must pass; the same battery must fail on
l = 1 (consecutive outputs are adjacent vertices) and on a plain 32-bit LCG
(low bits periodic) — proof that it has power.
"""
import numpy as np
import pytest

import battery as B
import oracle as O

M32 = 1 << 32
ALPHA = 1e-4  # per test; 22 p-values per run


def words(labels):
    """R12: the u32 stream is the little-endian words (x, y) of each label."""
    return np.ascontiguousarray(labels).reshape(-1).view(np.uint32)


@pytest.fixture(scope="module")
def c2_small():
    W, D = 4096, 256
    z = O.bulk(M32, 64, 64, 0x5EED0002, W, 0, W * D)
    return z, W, D


def test_oracle_passes_bulk_order(c2_small):
    z, W, D = c2_small
    res = B.run(words(z))
    bad = {k: v for k, v in res.items() if v < ALPHA}
    assert not bad, bad


def test_oracle_passes_walker_major_order(c2_small):
    z, W, D = c2_small
    res = B.run(words(z.reshape(D, W).T.copy()))
    bad = {k: v for k, v in res.items() if v < ALPHA}
    assert not bad, bad


def test_negative_control_l1_fails():
    W, D = 1024, 1024
    z = O.bulk(M32, 1, 64, 0x5EED0002, W, 0, W * D)
    res = B.run(words(z.reshape(D, W).T.copy()))
    failed = [k for k, v in res.items() if v < 1e-10]
    assert len(failed) >= 3, res


def test_battery_has_power_on_lcg():
    n = 1 << 20
    x = np.empty(n, dtype=np.uint64)
    s = 1
    for i in range(n):  # plain LCG x <- 69069 x + 1 mod 2^32
        s = (69069 * s + 1) & 0xFFFFFFFF
        x[i] = s
    res = B.run(x.astype(np.uint32))
    for k in ("birthday_spacings_lo", "hamming_indep", "random_walk"):
        assert res[k] < 1e-10, (k, res[k])


def test_battery_null_calibration():
    """On numpy's PCG64 the p-values are not systematically small."""
    ps = []
    for s in range(3):
        u = np.random.Generator(np.random.PCG64(s)).integers(0, M32, 1 << 21, dtype=np.uint64)
        ps += list(B.run(u.astype(np.uint32)).values())
    ps = np.array(ps)
    assert ps.min() > ALPHA and 0.3 < ps.mean() < 0.7


def test_gf2_rank_vs_xor_basis():
    """The vectorised elimination equals a plain xor-basis rank (Python ints)."""
    rng = np.random.default_rng(5)
    m = rng.integers(0, M32, (300, 32), dtype=np.uint64).astype(np.uint32)
    m[0] = 0
    m[1] = np.uint32(1) << np.arange(32, dtype=np.uint32)  # identity
    m[2, 16:] = m[2, :16]                                   # rank <= 16
    m[3] &= np.uint32(0xFF)                                 # rank <= 8

    def rank(rows):
        basis = {}  # leading bit -> vector with that leading bit
        for r in map(int, rows):
            while r:
                top = r.bit_length() - 1
                if top not in basis:
                    basis[top] = r
                    break
                r ^= basis[top]
        return len(basis)
    got = B._gf2_ranks(m)
    assert list(got) == [rank(r) for r in m]
    assert got[0] == 0 and got[1] == 32 and got[2] <= 16 and got[3] <= 8
