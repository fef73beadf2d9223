"""Pins for the Monte Carlo photon-migration oracle (§VI; no GPU).

The physics of photon migration is pinned by closed forms and a published
benchmark rather than by the oracle itself:
  * energy conservation is an exact integer identity (R22 fixed point);
  * a pure absorber with matched boundaries transmits e^{-mua d}
    (Beer-Lambert) and reflects nothing;
  * the Henyey-Greenstein sampler has mean cosine g;
  * Fresnel reflectance: normal-incidence closed form, total internal
    reflection beyond the critical angle, and reciprocity R(n1->n2, t1) =
    R(n2->n1, t2);
  * a semi-infinite, isotropically scattering medium under normal incidence
    reflects 1 - H(1) sqrt(1 - a) (Chandrasekhar's plane albedo; H is
    computed here from its integral equation, independently of the MC code).
"""
import math

import numpy as np
import pytest

import oracle as O


def frac(r, k):
    return r[k] / r["launched"]


@pytest.mark.parametrize("D", [3, 9, 192])
def test_energy_conservation_exact(D):
    r = O.mc_run(nthreads=64, photons_total=300, D=D, seed=3)
    tal = r["tallies"]
    assert tal[0] == tal[1:].sum()
    assert r["photons"] == 300
    assert abs(frac(r, "specular") - ((1 - 1.37) / (1 + 1.37)) ** 2) < 1e-9


def test_pure_absorber_beer_lambert():
    mua, d = 2.0, 0.5
    layers = [(1.0, mua, 0.0, 0.0, d)]
    P = 20000
    r = O.mc_run(layers=layers, nthreads=256, photons_total=P, D=12, seed=11)
    assert r["R_d"] == 0 and r["specular"] == 0 and r["terminated"] == 0
    t = frac(r, "T_t")
    want = math.exp(-mua * d)
    # weights W0 are independent of the path, so T_t/sum(W0) is an unbiased
    # estimate; binomial error with weight variance factor (E[W^2]/E[W]^2 = 4/3)
    sd = math.sqrt(want * (1 - want) / P * 4 / 3)
    assert abs(t - want) < 5 * sd
    assert r["interactions"] > 0  # absorbed photons drop all their weight at once
    assert r["launched"] == r["T_t"] + r["absorbed"][0]


@pytest.mark.parametrize("g", [0.0, 0.3, 0.75, 0.9, -0.5])
def test_hg_mean_cosine_is_g(g):
    xi = (np.arange(200000) + 0.5) / 200000
    c = np.array([O.mc_hg(g, v) for v in xi[::10]])
    assert abs(c.mean() - g) < 2e-4
    assert c.min() >= -1 and c.max() <= 1


def test_fresnel():
    n1, n2 = 1.0, 1.37
    r, ca2 = O.mc_fresnel(n1, n2, 1.0)
    assert abs(r - ((n2 - n1) / (n2 + n1)) ** 2) < 1e-15 and ca2 == 1.0
    assert O.mc_fresnel(1.37, 1.37, 0.3) == (0.0, 0.3)
    # total internal reflection beyond the critical angle, going 1.37 -> 1
    crit = math.sqrt(1 - (1 / 1.37) ** 2)   # cos of the critical angle
    assert O.mc_fresnel(1.37, 1.0, crit * 0.999)[0] == 1.0
    assert O.mc_fresnel(1.37, 1.0, crit * 1.01)[0] < 1.0
    # reciprocity: R(n1->n2, theta1) = R(n2->n1, theta2)
    for ca1 in (0.2, 0.5, 0.8, 0.95):
        r12, ca2 = O.mc_fresnel(n1, n2, ca1)
        r21, back = O.mc_fresnel(n2, n1, ca2)
        assert abs(r12 - r21) < 1e-12 and abs(back - ca1) < 1e-12
        assert 0 < r12 < 1


def chandrasekhar_H1(a, n=200):
    """H(mu=1) for isotropic scattering with albedo a, from
    H(mu) = 1 / (1 - (a/2) mu int_0^1 H(mu')/(mu + mu') dmu')  (Gauss-Legendre)."""
    x, w = np.polynomial.legendre.leggauss(n)
    mu, w = 0.5 * (x + 1), 0.5 * w
    H = np.ones(n)
    for _ in range(1000):
        Hn = 1.0 / (1.0 - 0.5 * a * mu * np.sum(w * H / (mu[:, None] + mu[None, :]), axis=1))
        if np.max(np.abs(Hn - H)) < 1e-14:
            break
        H = Hn
    return 1.0 / (1.0 - 0.5 * a * np.sum(w * H / (1.0 + mu)))


@pytest.mark.parametrize("a", [0.5, 0.9])
def test_semi_infinite_isotropic_albedo(a):
    mua = 1.0
    mus = mua * a / (1 - a)
    layers = [(1.0, mua, mus, 0.0, 1000.0 / (mua + mus))]  # optical depth 1000
    P = 40000
    r = O.mc_run(layers=layers, nthreads=512, photons_total=P, D=96, seed=2)
    want = 1 - chandrasekhar_H1(a) * math.sqrt(1 - a)
    sd = math.sqrt(want * (1 - want) / P * 4 / 3)
    assert abs(frac(r, "R_d") - want) < 4 * sd + frac(r, "terminated")
    assert r["T_t"] == 0


def test_r19_slab_plausible_and_threads_independent():
    # per-thread simulation: running threads in two shards sums to the whole
    a = O.mc_run(nthreads=128, photons_total=512, seed=5, per_thread=True)
    b1 = O.mc_run(nthreads=64, walker0=0, threads_total=128, photons_total=512, seed=5)
    b2 = O.mc_run(nthreads=64, walker0=64, threads_total=128, photons_total=512, seed=5)
    assert np.array_equal(a["tallies"], b1["tallies"] + b2["tallies"])
    assert np.array_equal(a["per_thread"].sum(axis=0), a["tallies"])
    assert 0.15 < frac(a, "R_d") < 0.35 and 0.05 < frac(a, "T_t") < 0.2
