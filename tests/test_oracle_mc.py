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
    computed here from its integral equation, independently of the MC code);
  * anisotropic transport (g = 0.75) in a finite slab: van de Hulst's
    tabulated R_d = 0.09739, T_t = 0.66096 for albedo 0.9, optical
    thickness 2, matched boundaries (the benchmark MCML was validated
    against: mua 10, mus 90 /cm, g 0.75, d 0.02 cm);
  * index-mismatched boundaries at normal incidence: a non-scattering slab
    between two ambient media transmits and reflects the geometric series of
    Fresnel bounces in closed form;
  * oblique refraction: the boundary-crossing step obeys Snell's law with a
    unit direction (or_mc_refract, the helper or_mc_run calls);
  * the scattering rotation (or_mc_spin) keeps |u| = 1, deflects by exactly
    the HG angle (u.u' = cos theta) and spreads the azimuth uniformly (slab
    tallies see only uz, so this is pinned on the helper itself).
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


def ratio_and_se(r, key):
    """Estimate sum(tally)/sum(launched) and its standard error from the
    per-thread rows (threads are iid: same photon budget, disjoint walkers)."""
    pt = r["per_thread"].astype(np.float64)
    k = 5 + int(key) if not isinstance(key, str) else O.MC_TALLY_NAMES.index(key)
    num, den = pt[:, k], pt[:, 0]
    est = num.sum() / den.sum()
    resid = num - est * den
    se = math.sqrt(resid.var(ddof=1) / len(den)) / den.mean()
    return est, se


def test_van_de_hulst_slab_g075():
    """Albedo 0.9, g = 0.75, optical thickness 2, n = 1 everywhere: van de
    Hulst's R_d = 0.09739 and T_t = 0.66096 (MCML's validation slab, mua 10,
    mus 90 /cm, d 0.02 cm).  Pins anisotropic HG transport, the hop / drop /
    spin loop and the direction update away from the normal."""
    layers = [(1.0, 10.0, 90.0, 0.75, 0.02)]
    r = O.mc_run(layers=layers, nthreads=1024, photons_total=300_000, D=96, seed=0x7A11,
                 per_thread=True)
    term = r["terminated"] / r["launched"]
    for key, want in (("R_d", 0.09739), ("T_t", 0.66096)):
        est, se = ratio_and_se(r, key)
        assert abs(est - want) < 4 * se + term, (key, est, want, se)
    assert r["specular"] == 0


@pytest.mark.parametrize("n_slab,n_bottom,tau", [(1.5, 1.0, 0.5), (1.37, 1.33, 1.0), (2.0, 1.0, 0.2)])
def test_mismatched_absorbing_slab_closed_form(n_slab, n_bottom, tau):
    """Pure absorber (mus = 0) of optical thickness tau, index n_slab, air
    above and n_bottom below, normal incidence.  The photon bounces between
    the faces; with R1 = ((1 - n)/(1 + n))^2 and R2 = ((n - n_b)/(n + n_b))^2
    the geometric series gives
        specular = R1,
        T_t = (1 - R1)(1 - R2) e^-tau / (1 - R1 R2 e^-2tau),
        R_d = (1 - R1)^2 R2 e^-2tau / (1 - R1 R2 e^-2tau)."""
    mua = 2.0
    layers = [(n_slab, mua, 0.0, 0.0, tau / mua)]
    r = O.mc_run(layers=layers, n_top=1.0, n_bottom=n_bottom, nthreads=1024,
                 photons_total=200_000, D=12, seed=0x3A5, per_thread=True)
    R1 = ((1 - n_slab) / (1 + n_slab)) ** 2
    R2 = ((n_slab - n_bottom) / (n_slab + n_bottom)) ** 2
    e1, e2 = math.exp(-tau), math.exp(-2 * tau)
    den = 1 - R1 * R2 * e2
    want = {"T_t": (1 - R1) * (1 - R2) * e1 / den, "R_d": (1 - R1) ** 2 * R2 * e2 / den}
    assert abs(r["specular"] / r["launched"] - R1) < 1e-9
    for key, w in want.items():
        est, se = ratio_and_se(r, key)
        assert abs(est - w) < 4 * se, (key, est, w, se)
    assert r["terminated"] == 0


def test_refraction_snell():
    """The transmitted direction (or_mc_refract, fed by or_mc_fresnel's
    cos(t2)) satisfies n1 sin t1 = n2 sin t2, stays a unit vector, keeps the
    plane of incidence and the direction of travel along z."""
    rng = np.random.default_rng(0x5E11)
    for n1, n2 in ((1.0, 1.37), (1.37, 1.0), (1.37, 1.5), (1.5, 1.33)):
        crit = 0.0 if n1 <= n2 else math.sqrt(1 - (n2 / n1) ** 2)  # cos of the critical angle
        done = 0
        while done < 200:
            v = rng.normal(size=3)
            v /= np.linalg.norm(v)
            if abs(v[2]) <= crit + 1e-6 or abs(v[2]) > 1 - 1e-9:
                continue
            _, ca2 = O.mc_fresnel(n1, n2, abs(v[2]))
            ux, uy, uz = O.mc_refract(n1, n2, ca2, v)
            s1 = math.hypot(v[0], v[1])
            s2 = math.hypot(ux, uy)
            assert abs(n1 * s1 - n2 * s2) < 1e-12
            assert abs(ux * ux + uy * uy + uz * uz - 1) < 1e-12
            assert abs(ux * v[1] - uy * v[0]) < 1e-12          # same plane of incidence
            assert ux * v[0] + uy * v[1] > 0 and uz * v[2] > 0   # no reversal
            done += 1
    # normal incidence passes straight through
    assert O.mc_refract(1.0, 1.5, 1.0, (0.0, 0.0, -1.0)) == (0.0, 0.0, -1.0)


def test_spin_rotation():
    rng = np.random.default_rng(0x5B1)
    for g in (0.0, 0.75, -0.4):
        for _ in range(300):
            v = rng.normal(size=3)
            v /= np.linalg.norm(v)
            if rng.random() < 0.1:  # the near-normal branch |uz| > 0.99999
                v = np.array([0.0, 0.0, 1.0 if rng.random() < 0.5 else -1.0])
            xt, xp = rng.random(), rng.random()
            u = np.array(O.mc_spin(g, xt, xp, v))
            assert abs(u @ u - 1) < 1e-12
            assert abs(u @ v - O.mc_hg(g, xt)) < 1e-12
    # azimuth: about u = e_z (psi measured from x) and about an oblique u the
    # deflected directions' components orthogonal to u average to zero
    for v in (np.array([0.0, 0.0, 1.0]), np.array([0.6, 0.0, 0.8]), np.array([0.0, -0.8, -0.6])):
        xs = (np.arange(4096) + 0.5) / 4096
        us = np.array([O.mc_spin(0.0, 0.3, xp, v) for xp in xs])
        perp = us - np.outer(us @ v, v)
        assert np.abs(perp.mean(axis=0)).max() < 1e-9
        # psi -> psi + pi reflects the perpendicular part
        a = np.array(O.mc_spin(0.0, 0.3, 0.1, v))
        b = np.array(O.mc_spin(0.0, 0.3, 0.6, v))
        pa, pb = a - (a @ v) * v, b - (b @ v) * v
        assert np.abs(pa + pb).max() < 1e-12
