"""More empirical tests in the style of TestU01 Crush (test infrastructure
only; SURVEY §8(f) f4 — the paper reports Crush-level results, §IV-B
Table III).  Each is written from its textbook definition with an exact null
distribution:

  runs_up     Knuth TAOCP 3.3.2 G, the variant that discards the element
              after each run so run lengths are independent:
              P(length = r) = r / (r+1)!                          (sknuth_Run)
  gcd         Marsaglia & Tsang (2002): gcd of two random 32-bit words,
              P(gcd = j) -> 6 / (pi^2 j^2)                        (smarsa_GCD)
  autocor     XOR of bits d apart: sum ~ Binomial(n - d, 1/2)    (sstring_AutoCor)
  sample_prod -ln(U_1 ... U_t) ~ Gamma(t, 1), KS test         (svaria_SampleProd)

Each function takes uint32 words and returns a p-value.
"""
from __future__ import annotations

import math

import numpy as np
from scipy import stats

from battery import _chi2, _uniform


def runs_up_probs(kmax):
    """P(run length = r) for r = 1..kmax-1 and P(>= kmax), the discard variant."""
    p = [r / math.factorial(r + 1) for r in range(1, kmax)]
    return p + [1.0 - sum(p)]


def runs_up(u, kmax=7):
    """Run-up lengths of U = word / 2^32, skipping the element after each run."""
    x = _uniform(u)
    n = x.size
    lengths = []
    i = 0
    # vectorised scan: positions where the sequence stops increasing
    desc = np.flatnonzero(x[1:] <= x[:-1])  # run ends at index d (x[d+1] <= x[d])
    j = 0
    while i < n - 1:
        k = np.searchsorted(desc, i)        # first descent at or after i
        if k >= desc.size:
            break
        end = int(desc[k])                  # run is x[i..end]
        lengths.append(end - i + 1)
        i = end + 2                         # discard x[end + 1]
        j += 1
    L = np.minimum(np.array(lengths), kmax) - 1
    return _chi2(np.bincount(L, minlength=kmax), runs_up_probs(kmax))


def gcd_probs(jmax):
    """P(gcd = j) = 6 / (pi^2 j^2) for j < jmax, the rest pooled."""
    p = [6.0 / (math.pi ** 2 * j * j) for j in range(1, jmax)]
    return p + [1.0 - sum(p)]


def gcd(u, jmax=40):
    a = u[0::2].astype(np.int64)
    b = u[1::2].astype(np.int64)
    m = min(a.size, b.size)
    a, b = a[:m], b[:m]
    keep = (a > 0) & (b > 0)
    g = np.gcd(a[keep], b[keep])
    return _chi2(np.bincount(np.minimum(g, jmax) - 1, minlength=jmax), gcd_probs(jmax))


def autocor(u, d=1, nbits=1 << 22):
    """Bits (MSB first) of the words; A = sum b_i xor b_(i+d); two-sided."""
    b = np.unpackbits(np.ascontiguousarray(u, dtype=np.uint32).byteswap().view(np.uint8))[:nbits]
    n = b.size - d
    a = int(np.count_nonzero(b[:-d] != b[d:]))
    z = (a - n / 2.0) / math.sqrt(n / 4.0)
    return float(2 * stats.norm.sf(abs(z)))


def sample_prod(u, t=8):
    x = _uniform(u)
    m = x.size // t
    s = -np.log(x[: m * t].reshape(m, t)).sum(axis=1)
    return float(stats.kstest(s, stats.gamma(t).cdf).pvalue)


def run(u):
    u = np.ascontiguousarray(u, dtype=np.uint32).reshape(-1)
    return {
        "runs_up": runs_up(u[: 1 << 20]),
        "gcd": gcd(u),
        "autocor_1": autocor(u, 1),
        "autocor_8": autocor(u, 8),
        "autocor_32": autocor(u, 32),
        "autocor_64": autocor(u, 64),
        "sample_prod": sample_prod(u),
    }
