"""Statistical pins for the oracle on config C1 (P7-P9, with negative controls).

Config C1 (BASELINE.json configs[0]): m = 2^8, degree 7, l = l0 = 64,
W = 1024 walkers, 2^20 numbers, seed 0x5EED0001.

The exact null holds by P3 (uniform is stationary, each output uniform), and
the walk of l = 64 steps leaves a chi^2-divergence of ~2e-16 between
consecutive outputs, so every test must pass at alpha = 1e-3.
Negative controls prove the tests have power: at l = 16 the parity-pair
projection must fail (divergence 2(3/4)^32 + (1/2)^32 ~ 2e-4, N*D ~ 210 vs a
critical value of 37.7) and at l = 1 every test fails.  Quality claims in the
paper: DIEHARD/TestU01 (§IV-B, Tables II-III).
"""
import numpy as np
import pytest
from scipy import stats

import oracle as O

M, W, SEED = 256, 1024, 0x5EED0001
ALPHA = 1e-3


@pytest.fixture(scope="module")
def c1_l64():
    return O.bulk(M, 64, 64, SEED, W, 0, 1 << 20).astype(np.int64)


def _chi2_p(counts, expected):
    chi = ((counts - expected) ** 2 / expected).sum()
    return stats.chi2.sf(chi, counts.size - 1), chi


def equidistribution_p(z):
    return _chi2_p(np.bincount(z, minlength=M * M).astype(float), z.size / (M * M))[0]


def serial_parity_p(z):
    """Pairs (v_j, v_{j+1}) of the same walker, projected on (x mod 2, y mod 2)^2."""
    zz = z.reshape(-1, W)  # [draw, walker]
    a, b = zz[:-1].ravel(), zz[1:].ravel()
    cell = lambda v: (v % M) % 2 + 2 * ((v // M) % 2)
    c = cell(a) * 4 + cell(b)
    return _chi2_p(np.bincount(c, minlength=16).astype(float), c.size / 16)


def serial_mod4_p(z):
    zz = z.reshape(-1, W)
    a, b = zz[:-1].ravel(), zz[1:].ravel()
    cell = lambda v: (v % M) % 4 + 4 * ((v // M) % 4)
    c = cell(a) * 16 + cell(b)
    return _chi2_p(np.bincount(c, minlength=256).astype(float), c.size / 256)[0]


def serial_top_p(z):
    zz = z.reshape(-1, W)
    a, b = zz[:-1].ravel(), zz[1:].ravel()
    cell = lambda v: ((v % M) >> 6) + 4 * ((v // M) >> 6)
    c = cell(a) * 16 + cell(b)
    return _chi2_p(np.bincount(c, minlength=256).astype(float), c.size / 256)[0]


def gap_p(indicator):
    """Knuth's gap test: lengths of runs between hits of an event of prob 1/2,
    gaps >= 10 pooled."""
    idx = np.flatnonzero(indicator)
    gaps = np.diff(idx) - 1
    gaps = np.minimum(gaps, 10)
    counts = np.bincount(gaps, minlength=11).astype(float)
    p = np.array([0.5 ** (g + 1) for g in range(10)] + [0.5 ** 10])
    return _chi2_p(counts, p * gaps.size)[0]


def test_p7_equidistribution(c1_l64):
    z = c1_l64
    assert equidistribution_p(z) > ALPHA
    # 256-cell projections on the low 8 bits (x) and the top 8 bits (y)
    assert _chi2_p(np.bincount(z % M, minlength=M).astype(float), z.size / M)[0] > ALPHA
    assert _chi2_p(np.bincount(z // M, minlength=M).astype(float), z.size / M)[0] > ALPHA


def test_p8_serial(c1_l64):
    assert serial_parity_p(c1_l64)[0] > ALPHA
    assert serial_mod4_p(c1_l64) > ALPHA
    assert serial_top_p(c1_l64) > ALPHA


def test_p9_gap(c1_l64):
    z = c1_l64
    assert gap_p(z < (M * M) // 2) > ALPHA          # u = label / m^2 in [0, 1/2)
    assert gap_p(((z // M) >> 7) == 1) > ALPHA      # top bit of the label


def test_negative_control_l16_fails_parity_serial():
    z = O.bulk(M, 16, 64, SEED, W, 0, 1 << 20).astype(np.int64)
    p, chi = serial_parity_p(z)
    assert p < 1e-10, chi
    assert chi > 100  # expected N*D ~ 210 + 15 dof


def test_negative_control_l1_fails_everything():
    z = O.bulk(M, 1, 64, SEED, W, 0, 1 << 18).astype(np.int64)
    assert serial_parity_p(z)[0] < 1e-10
    assert serial_mod4_p(z) < 1e-10
    assert serial_top_p(z) < 1e-10
