"""Crush-style tests (tests/battery_crush.py): null distributions pinned by
brute force and closed forms, then run on the oracle's C2-type output with
negative controls (§IV-B Table III)."""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest

import battery_crush as C
import oracle as O

M32 = 1 << 32
ALPHA = 1e-4


def test_runs_up_law_by_enumeration():
    # first run-up length of 7 distinct values: P(len = r) = r / (r+1)!
    n = 7
    cnt = [0] * (n + 1)
    for p in itertools.permutations(range(n)):
        r = 1
        while r < n and p[r] > p[r - 1]:
            r += 1
        cnt[r] += 1
    tot = math.factorial(n)
    for r in range(1, n):
        assert Fraction(cnt[r], tot) == Fraction(r, math.factorial(r + 1))
    assert sum(C.runs_up_probs(7)) == pytest.approx(1.0, abs=1e-15)


def test_gcd_law():
    assert sum(6 / (math.pi ** 2 * j * j) for j in range(1, 200000)) == pytest.approx(1.0, abs=1e-5)
    # brute force over all pairs in [1, 2000]^2
    a = np.arange(1, 2001)
    g = np.gcd(a[:, None], a[None, :]).ravel()
    f = np.bincount(g, minlength=6)[1:6] / g.size
    assert np.allclose(f, C.gcd_probs(40)[:5], atol=2e-3)


def test_autocor_and_sample_prod_have_power():
    rng = np.random.default_rng(3)
    u = rng.integers(0, M32, 1 << 18, dtype=np.uint64).astype(np.uint32)
    assert C.autocor(u, 8) > ALPHA and C.sample_prod(u) > ALPHA
    rep = np.repeat(u[: 1 << 17], 2)          # every word twice: bits 32 apart agree
    assert C.autocor(rep, 32) < 1e-10
    sq = (u.astype(np.uint64) * u.astype(np.uint64) >> 32).astype(np.uint32)  # U^2 law, not U
    assert C.sample_prod(sq) < 1e-10


@pytest.fixture(scope="module")
def c2_words():
    W, D = 4096, 256
    z = O.bulk(M32, 64, 64, 0x5EED0002, W, 0, W * D)
    return z, W, D


def test_oracle_passes(c2_words):
    z, W, D = c2_words
    for arr in (z, z.reshape(D, W).T.copy()):
        res = C.run(np.ascontiguousarray(arr).reshape(-1).view(np.uint32))
        bad = {k: v for k, v in res.items() if v < ALPHA}
        assert not bad, bad


def test_negative_controls():
    # plain LCG x <- 69069 x + 1: the low bit alternates, so a pair's gcd is never even
    n = 1 << 20
    x = np.empty(n, dtype=np.uint64)
    s = 1
    for i in range(n):
        s = (69069 * s + 1) & 0xFFFFFFFF
        x[i] = s
    assert C.gcd(x.astype(np.uint32)) < 1e-10
    # l = 1 walker-major: consecutive outputs are adjacent vertices
    W, D = 1024, 1024
    z = O.bulk(M32, 1, 64, 0x5EED0002, W, 0, W * D)
    res = C.run(np.ascontiguousarray(z.reshape(D, W).T).reshape(-1).view(np.uint32))
    assert sum(v < 1e-10 for v in res.values()) >= 2, res


def test_null_calibration():
    ps = []
    for s in range(3):
        u = np.random.Generator(np.random.PCG64(100 + s)).integers(0, M32, 1 << 21, dtype=np.uint64)
        ps += list(C.run(u.astype(np.uint32)).values())
    ps = np.array(ps)
    assert ps.min() > ALPHA and 0.25 < ps.mean() < 0.75
