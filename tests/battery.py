"""A small empirical-test battery in the style of TestU01 SmallCrush (test
infrastructure only).

The paper validates its generator with DIEHARD and TestU01 (§IV-B,
Tables II-III).  Neither suite is available offline, so this module
re-implements, from their textbook definitions (Knuth TAOCP vol. 2 §3.3.2;
Marsaglia's birthday spacings; L'Ecuyer & Simard's SmallCrush list), the
tests that SmallCrush is made of, with exact or standard asymptotic null
distributions:

  birthday_spacings  (smarsa_BirthdaySpacings)  Y ~ Poisson(m^3 / 4n)
  collision          (sknuth_Collision)          C ~ Poisson(E[C])
  gap                (sknuth_Gap)                geometric gap lengths
  simple_poker       (sknuth_SimpPoker)          Stirling numbers of 2nd kind
  coupon_collector   (sknuth_CouponCollector)    d!/d^r S(r-1, d-1)
  max_of_t           (sknuth_MaxOft)             max^t ~ U(0,1)
  weight_distrib     (svaria_WeightDistrib)      Binomial(k, beta)
  matrix_rank        (smarsa_MatrixRank)         GF(2) rank law of L x L
  hamming_indep      (sstring_HammingIndep)      independence of popcounts
  random_walk        (swalk_RandomWalk1)         final position of a +-1 walk

Every function takes a 1-D array of uint32 words and returns a p-value
(two-sided where the statistic can err both ways).  Inputs never come from
the code under test's own arithmetic: the battery only reads the words.
"""
from __future__ import annotations

import math

import numpy as np
from scipy import stats


def _chi2(counts, probs, min_expected=5.0):
    """Chi-square p-value of `counts` against cell probabilities `probs`,
    merging adjacent small cells until each expected count >= min_expected."""
    counts = np.asarray(counts, dtype=float)
    probs = np.asarray(probs, dtype=float)
    n = counts.sum()
    exp = probs * n
    oc, ec = [], []
    acc_o = acc_e = 0.0
    for o, e in zip(counts, exp):
        acc_o += o
        acc_e += e
        if acc_e >= min_expected:
            oc.append(acc_o)
            ec.append(acc_e)
            acc_o = acc_e = 0.0
    if acc_e > 0 and ec:
        oc[-1] += acc_o
        ec[-1] += acc_e
    oc, ec = np.array(oc), np.array(ec)
    if oc.size < 2:
        return 1.0
    chi = ((oc - ec) ** 2 / ec).sum()
    return float(stats.chi2.sf(chi, oc.size - 1))


def _poisson_two_sided(x, lam):
    lo = stats.poisson.cdf(x, lam)
    hi = stats.poisson.sf(x - 1, lam)
    return float(min(1.0, 2 * min(lo, hi)))


def _uniform(u):
    return (u.astype(np.float64) + 0.5) / 2.0 ** 32


def birthday_spacings(u, bits=24, shift=8, m=512, reps=None):
    """Marsaglia: m birthdays in a year of n = 2^bits days (bits of each word
    taken from bit `shift` up); Y = number of repeated values among the
    sorted spacings, summed over reps, ~ Poisson(reps * m^3 / (4n))."""
    reps = reps or u.size // m
    v = ((u[: reps * m] >> np.uint32(shift)) & np.uint32((1 << bits) - 1)).astype(np.int64)
    v = np.sort(v.reshape(reps, m), axis=1)
    sp = np.sort(np.diff(v, axis=1, prepend=0), axis=1)
    y = int((sp[:, 1:] == sp[:, :-1]).sum())
    lam = reps * m ** 3 / (4.0 * 2 ** bits)
    return _poisson_two_sided(y, lam)


def collision(u, t=2, bits=15, n=1 << 16, reps=None):
    """Knuth: n points of t consecutive `bits`-bit values (top bits) thrown into
    k = 2^(t*bits) cells; collisions summed over reps ~ Poisson(reps*E[C])."""
    k = 2.0 ** (t * bits)
    reps = reps or max(1, u.size // (n * t))
    v = (u[: reps * n * t] >> np.uint32(32 - bits)).astype(np.int64).reshape(reps, n, t)
    cell = np.zeros((reps, n), dtype=np.int64)
    for i in range(t):
        cell = (cell << bits) | v[:, :, i]
    c = 0
    for r in range(reps):
        c += n - np.unique(cell[r]).size
    ec = n - k * (1.0 - math.exp(n * math.log1p(-1.0 / k)))
    return _poisson_two_sided(c, reps * ec)


def gap(u, alpha=0.0, beta=0.125, t=30):
    """Knuth's gap test on U = word/2^32 with the interval [alpha, beta):
    gap lengths r = 0..t-1 with P = p(1-p)^r, r >= t pooled."""
    x = _uniform(u)
    hit = np.flatnonzero((x >= alpha) & (x < beta))
    g = np.minimum(np.diff(hit) - 1, t)
    p = beta - alpha
    probs = [p * (1 - p) ** r for r in range(t)] + [(1 - p) ** t]
    return _chi2(np.bincount(g, minlength=t + 1), probs)


def _stirling2(n, k):
    s = [[0] * (k + 1) for _ in range(n + 1)]
    s[0][0] = 1
    for i in range(1, n + 1):
        for j in range(1, min(i, k) + 1):
            s[i][j] = j * s[i - 1][j] + s[i - 1][j - 1]
    return s[n][k]


def simple_poker(u, d=16, k=8):
    """Knuth's simplified poker: groups of k values in d categories (top bits);
    number of distinct values r has P = d(d-1)..(d-r+1)/d^k * S(k, r)."""
    b = int(math.log2(d))
    v = (u[: (u.size // k) * k] >> np.uint32(32 - b)).reshape(-1, k).astype(np.int64)
    onehot = np.zeros((v.shape[0], d), dtype=bool)
    np.put_along_axis(onehot, v, True, axis=1)
    r = onehot.sum(axis=1)
    probs = []
    for rr in range(1, k + 1):
        falling = 1.0
        for i in range(rr):
            falling *= (d - i)
        probs.append(falling / d ** k * _stirling2(k, rr))
    return _chi2(np.bincount(r, minlength=k + 1)[1:], probs)


def coupon_collector(u, d=8, t=40):
    """Knuth: lengths of segments needed to collect all d categories (top
    bits); P(r) = d!/d^r S(r-1, d-1) for d <= r < t, r >= t pooled."""
    b = int(math.log2(d))
    v = (u >> np.uint32(32 - b)).astype(np.int64)
    lengths = []
    seen = 0
    count = 0
    full = (1 << d) - 1
    # plain loop over a bounded prefix (segments are ~22 values long)
    for c in v[: min(v.size, 1 << 20)]:
        seen |= 1 << int(c)
        count += 1
        if seen == full:
            lengths.append(count)
            seen = 0
            count = 0
    L = np.minimum(np.array(lengths), t)
    fact = math.factorial(d)
    probs = [fact / d ** r * _stirling2(r - 1, d - 1) for r in range(d, t)]
    probs.append(1.0 - sum(probs))
    return _chi2(np.bincount(L - d, minlength=t - d + 1), probs)


def max_of_t(u, t=8, cells=100):
    """Knuth: V = max of t uniforms; V^t ~ U(0,1), chi-square over `cells`."""
    x = _uniform(u[: (u.size // t) * t]).reshape(-1, t).max(axis=1) ** t
    return _chi2(np.bincount(np.minimum((x * cells).astype(int), cells - 1), minlength=cells),
                 [1.0 / cells] * cells)


def weight_distrib(u, k=256, beta=0.25):
    """L'Ecuyer: number of the k uniforms of a block in [0, beta) ~ Bin(k, beta)."""
    x = _uniform(u[: (u.size // k) * k]).reshape(-1, k)
    w = (x < beta).sum(axis=1)
    return _chi2(np.bincount(w, minlength=k + 1), stats.binom.pmf(np.arange(k + 1), k, beta))


def _gf2_ranks(rows):
    """Ranks over GF(2) of a batch of 32x32 bit matrices (rows: [N, 32] uint32)."""
    a = rows.astype(np.uint64).copy()
    N = a.shape[0]
    rank = np.zeros(N, dtype=np.int64)
    active = np.ones((N, 32), dtype=bool)  # rows not yet used as pivots
    for bit in range(31, -1, -1):
        has = ((a >> np.uint64(bit)) & np.uint64(1)).astype(bool) & active
        piv_exists = has.any(axis=1)
        piv = np.argmax(has, axis=1)
        idx = np.flatnonzero(piv_exists)
        prow = a[idx, piv[idx]]
        # eliminate the bit from every other row that has it
        elim = has[idx].copy()
        elim[np.arange(idx.size), piv[idx]] = False
        a[idx] ^= np.where(elim, prow[:, None], np.uint64(0))
        active[idx, piv[idx]] = False
        rank[idx] += 1
    return rank


def matrix_rank(u, L=32):
    """Marsaglia: rank over GF(2) of L x L matrices (32 consecutive words);
    P(r) = 2^(r(2L-r)-L^2) prod_{i<r} (1-2^(i-L))^2 / (1-2^(i-r))."""
    assert L == 32
    m = u[: (u.size // 32) * 32].reshape(-1, 32)
    r = _gf2_ranks(m)

    def p(rr):
        v = 2.0 ** (rr * (2 * L - rr) - L * L)
        for i in range(rr):
            v *= (1 - 2.0 ** (i - L)) ** 2 / (1 - 2.0 ** (i - rr))
        return v
    ranks = np.arange(29, 33)
    probs = [sum(p(rr) for rr in range(0, 30))] + [p(rr) for rr in ranks[1:]]
    counts = [np.sum(r <= 29)] + [np.sum(r == rr) for rr in ranks[1:]]
    return _chi2(counts, probs, min_expected=1.0)


def hamming_indep(u, cats=(13, 14, 15, 16, 17, 18, 19)):
    """Popcounts of consecutive words, binned (<=13, 14..18, >=19), tested for
    independence against the product of Binomial(32, 1/2) marginals."""
    w = np.unpackbits(u.view(np.uint8)).reshape(-1, 32).sum(axis=1)
    edges = np.array(cats)
    b = np.searchsorted(edges, w, side="left")  # 0: <=13 ... len(cats): >=20
    nb = edges.size + 1
    pm = np.array([stats.binom.cdf(cats[0], 32, 0.5)] +
                  [stats.binom.pmf(c, 32, 0.5) for c in cats[1:]] +
                  [stats.binom.sf(cats[-1], 32, 0.5)])
    a, c = b[0:-1:2], b[1::2]  # disjoint pairs
    cell = a * nb + c
    return _chi2(np.bincount(cell, minlength=nb * nb), np.outer(pm, pm).ravel())


def random_walk(u, steps=1024):
    """Final position of a +-1 walk driven by the bits of steps/32 words:
    (S + steps)/2 ~ Binomial(steps, 1/2)."""
    wpw = steps // 32
    v = u[: (u.size // wpw) * wpw].reshape(-1, wpw)
    ones = np.unpackbits(v.view(np.uint8), axis=1).sum(axis=1)
    return _chi2(np.bincount(ones, minlength=steps + 1),
                 stats.binom.pmf(np.arange(steps + 1), steps, 0.5))


def run(u, scale=1.0):
    """The battery on uint32 words `u`; returns {test name: p-value}."""
    u = np.ascontiguousarray(u, dtype=np.uint32).reshape(-1)
    res = {
        "birthday_spacings_hi": birthday_spacings(u, bits=24, shift=8),
        "birthday_spacings_lo": birthday_spacings(u, bits=24, shift=0),
        "collision": collision(u),
        "gap": gap(u),
        "simple_poker": simple_poker(u),
        "coupon_collector": coupon_collector(u),
        "max_of_t": max_of_t(u),
        "weight_distrib": weight_distrib(u),
        "matrix_rank": matrix_rank(u),
        "hamming_indep": hamming_indep(u),
        "random_walk": random_walk(u),
    }
    return res
