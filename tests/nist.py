"""NIST SP 800-22 statistical tests (test infrastructure only).

A second, independent family of empirical tests next to the SmallCrush-style
battery (tests/battery.py).  The paper validates its generator with DIEHARD
and TestU01 (§IV-B); neither suite is available offline.  These are the
bit-level tests of NIST SP 800-22 rev. 1a (Rukhin et al., 2010), written from
the test definitions in §2 of that document:

  frequency              2.1  monobit
  block_frequency        2.2  frequency within M-bit blocks
  runs                   2.3  number of runs
  longest_run            2.4  longest run of ones in a block
  dft                    2.6  discrete Fourier transform (spectral)
  linear_complexity      2.10 Berlekamp-Massey over M-bit blocks
  serial                 2.11 overlapping m-bit patterns (two p-values)
  approximate_entropy    2.12
  cumulative_sums        2.13 forward and backward

Each function takes a 1-D uint8 array of bits (0/1) and returns a p-value (or
a tuple of p-values).  `bits_of_words` turns uint32 words into bits, most
significant bit first.  The worked examples of SP 800-22 pin the arithmetic
(tests/test_nist.py); linear complexity is also pinned against sequences of
known complexity (LFSR outputs).
"""
from __future__ import annotations

import math

import numpy as np
from scipy import special


def bits_of_words(u):
    """uint32 words -> bits, MSB first within each word."""
    u = np.ascontiguousarray(u, dtype=np.uint32).reshape(-1)
    b = u.byteswap().view(np.uint8)  # big-endian bytes
    return np.unpackbits(b)


def bits_of_string(s: str):
    return np.frombuffer(s.encode(), dtype=np.uint8) - ord("0")


def _igamc(a, x):
    return float(special.gammaincc(a, x))


def frequency(e):
    """2.1: S_n = sum(2e - 1); P = erfc(|S_n| / sqrt(2n))."""
    n = e.size
    s = 2 * int(e.sum()) - n
    return float(special.erfc(abs(s) / math.sqrt(n) / math.sqrt(2)))


def block_frequency(e, M=128):
    """2.2: chi2 = 4M sum (pi_i - 1/2)^2 over N = n // M blocks; P = igamc(N/2, chi2/2)."""
    N = e.size // M
    pi = e[:N * M].reshape(N, M).sum(axis=1) / M
    chi2 = 4.0 * M * float(((pi - 0.5) ** 2).sum())
    return _igamc(N / 2.0, chi2 / 2.0)


def runs(e):
    """2.3: V_n = 1 + #{k : e_k != e_k+1}; P = erfc(|V - 2n pi (1-pi)| / (2 sqrt(2n) pi (1-pi)))."""
    n = e.size
    pi = float(e.sum()) / n
    if abs(pi - 0.5) >= 2.0 / math.sqrt(n):  # frequency prerequisite fails
        return 0.0
    v = 1 + int(np.count_nonzero(e[1:] != e[:-1]))
    num = abs(v - 2.0 * n * pi * (1 - pi))
    den = 2.0 * math.sqrt(2.0 * n) * pi * (1 - pi)
    return float(special.erfc(num / den))


_LONGEST = {  # M: (K, classes v <= lo, lo+1, ..., v >= hi) — SP 800-22 §2.4.2
    8: (3, 1, 4),
    128: (5, 4, 9),
    10000: (6, 10, 16),
}


def longest_run_class_probs(M, lo, hi):
    """Exact P(class) of the longest run of ones in M fair bits, by dynamic
    programming over the current run length (the probability tables of
    SP 800-22 §3.4 are these values rounded to 4 digits; its worked example
    uses the exact M = 8 values 55/256, 94/256, 59/256, 48/256)."""
    def p_le(k):  # P(longest run <= k)
        st = np.zeros(k + 1)
        st[0] = 1.0
        for _ in range(M):
            nxt = np.zeros(k + 1)
            nxt[0] = 0.5 * st.sum()          # a zero resets the run
            nxt[1:] = 0.5 * st[:-1]          # a one extends it (runs > k are dropped)
            st = nxt
        return float(st.sum())
    cdf = [p_le(k) for k in range(lo, hi)]
    probs = [cdf[0]] + [cdf[i] - cdf[i - 1] for i in range(1, len(cdf))] + [1.0 - cdf[-1]]
    return np.array(probs)


def _longest_run_ones(blocks):
    """Longest run of ones in each row of a 0/1 matrix."""
    best = np.zeros(blocks.shape[0], dtype=np.int64)
    cur = np.zeros(blocks.shape[0], dtype=np.int64)
    for j in range(blocks.shape[1]):
        col = blocks[:, j].astype(np.int64)
        cur = (cur + 1) * col
        np.maximum(best, cur, out=best)
    return best


def longest_run(e):
    """2.4: longest run of ones in M-bit blocks, chi2 over K+1 classes."""
    n = e.size
    M = 8 if n < 6272 else (128 if n < 750000 else 10000)
    K, lo, hi = _LONGEST[M]
    N = n // M
    v = _longest_run_ones(e[:N * M].reshape(N, M))
    v = np.clip(v, lo, hi) - lo
    counts = np.bincount(v, minlength=K + 1)
    pis = longest_run_class_probs(M, lo, hi)
    chi2 = float((((counts - N * pis) ** 2) / (N * pis)).sum())
    return _igamc(K / 2.0, chi2 / 2.0)


def dft(e):
    """2.6: |FFT(2e - 1)| below T = sqrt(ln(1/0.05) n) for the first n/2 terms;
    d = (N1 - 0.95 n/2) / sqrt(n 0.95 0.05 / 4); P = erfc(|d| / sqrt(2))."""
    n = e.size
    x = 2.0 * e.astype(np.float64) - 1.0
    m = np.abs(np.fft.fft(x))[: n // 2]
    T = math.sqrt(math.log(1.0 / 0.05) * n)
    n0 = 0.95 * n / 2.0
    n1 = float(np.count_nonzero(m < T))
    d = (n1 - n0) / math.sqrt(n * 0.95 * 0.05 / 4.0)
    return float(special.erfc(abs(d) / math.sqrt(2)))


def berlekamp_massey(blocks):
    """Linear complexity of each row of a 0/1 matrix (GF(2) Berlekamp-Massey,
    vectorised across rows): C(x) the current connection polynomial, B(x) the
    one before the last length change at position m."""
    blocks = np.asarray(blocks, dtype=np.uint8)
    R, M = blocks.shape
    C = np.zeros((R, M + 1), dtype=np.uint8)
    B = np.zeros((R, M + 1), dtype=np.uint8)
    C[:, 0] = 1
    B[:, 0] = 1
    L = np.zeros(R, dtype=np.int64)
    m = np.full(R, -1, dtype=np.int64)
    for N in range(M):
        # discrepancy d = s_N + sum_{i=1..L} C_i s_{N-i}  (C_i = 0 for i > L)
        d = (C[:, : N + 1] & blocks[:, N::-1]).sum(axis=1) & 1
        rows = np.nonzero(d)[0]
        if rows.size == 0:
            continue
        T = C[rows].copy()
        shift = N - m[rows]  # C <- C + x^(N - m) B
        for sh in np.unique(shift):
            r = rows[shift == sh]
            C[r, sh:] ^= B[r, : M + 1 - sh]
        grow = 2 * L[rows] <= N
        g = rows[grow]
        L[g] = N + 1 - L[g]
        m[g] = N
        B[g] = T[grow]
    return L


def linear_complexity(e, M=500):
    """2.10: T_i = (-1)^M (L_i - mu) + 2/9 binned into 7 classes; P = igamc(3, chi2/2)."""
    N = e.size // M
    L = berlekamp_massey(e[:N * M].reshape(N, M)).astype(np.float64)
    mu = M / 2.0 + (9 + (-1) ** (M + 1)) / 36.0 - (M / 3.0 + 2.0 / 9.0) / 2.0 ** M
    T = (-1) ** M * (L - mu) + 2.0 / 9.0
    edges = [-2.5, -1.5, -0.5, 0.5, 1.5, 2.5]
    v = np.searchsorted(edges, T, side="right")  # <= -2.5 -> 0 ... > 2.5 -> 6
    counts = np.bincount(v, minlength=7)
    pis = np.array([0.010417, 0.03125, 0.125, 0.5, 0.25, 0.0625, 0.020833])
    chi2 = float((((counts - N * pis) ** 2) / (N * pis)).sum())
    return _igamc(3.0, chi2 / 2.0)


def _psi2(e, m):
    """psi^2_m = 2^m / n sum_i v_i^2 - n over overlapping m-bit patterns (wrapping)."""
    n = e.size
    if m <= 0:
        return 0.0
    ext = np.concatenate([e, e[: m - 1]]).astype(np.int64)
    code = np.zeros(n, dtype=np.int64)
    for j in range(m):
        code = (code << 1) | ext[j:j + n]
    v = np.bincount(code, minlength=1 << m).astype(np.float64)
    return float((1 << m) / n * (v * v).sum() - n)


def serial(e, m=16):
    """2.11: P1 = igamc(2^(m-2), del psi^2 / 2), P2 = igamc(2^(m-3), del^2 psi^2 / 2)."""
    p0, p1, p2 = _psi2(e, m), _psi2(e, m - 1), _psi2(e, m - 2)
    d1 = p0 - p1
    d2 = p0 - 2 * p1 + p2
    return _igamc(2.0 ** (m - 2), d1 / 2.0), _igamc(2.0 ** (m - 3), d2 / 2.0)


def _phi(e, m):
    n = e.size
    ext = np.concatenate([e, e[: m - 1]]).astype(np.int64) if m > 1 else e.astype(np.int64)
    code = np.zeros(n, dtype=np.int64)
    for j in range(m):
        code = (code << 1) | ext[j:j + n]
    c = np.bincount(code, minlength=1 << m).astype(np.float64) / n
    c = c[c > 0]
    return float((c * np.log(c)).sum())


def approximate_entropy(e, m=10):
    """2.12: ApEn = phi(m) - phi(m+1); chi2 = 2n (ln 2 - ApEn); P = igamc(2^(m-1), chi2/2)."""
    n = e.size
    apen = _phi(e, m) - _phi(e, m + 1)
    chi2 = 2.0 * n * (math.log(2) - apen)
    return _igamc(2.0 ** (m - 1), chi2 / 2.0)


def _tdiv(a, b):
    """Integer division truncating toward zero (C semantics of the reference code)."""
    q = abs(a) // abs(b)
    return q if (a >= 0) == (b > 0) else -q


def cumulative_sums(e, reverse=False):
    """2.13: z = max_k |S_k| of the +-1 walk (forward or backward);
    P = 1 - sum_k [Phi((4k+1)z/sqrt n) - Phi((4k-1)z/sqrt n)]
          + sum_k [Phi((4k+3)z/sqrt n) - Phi((4k+1)z/sqrt n)]."""
    n = e.size
    x = 2 * e.astype(np.int64) - 1
    if reverse:
        x = x[::-1]
    z = int(np.abs(np.cumsum(x)).max())
    if z == 0:
        return 0.0
    Phi = lambda t: 0.5 * special.erfc(-t / math.sqrt(2))  # noqa: E731
    sq = math.sqrt(n)
    s1 = sum(Phi((4 * k + 1) * z / sq) - Phi((4 * k - 1) * z / sq)
             for k in range(_tdiv(_tdiv(-n, z) + 1, 4), _tdiv(_tdiv(n, z) - 1, 4) + 1))
    s2 = sum(Phi((4 * k + 3) * z / sq) - Phi((4 * k + 1) * z / sq)
             for k in range(_tdiv(_tdiv(-n, z) - 3, 4), _tdiv(_tdiv(n, z) - 1, 4) + 1))
    return float(1.0 - s1 + s2)


def run(bits):
    """The suite on one bit sequence (>= 10^6 bits recommended); {name: p-value}."""
    e = np.ascontiguousarray(bits, dtype=np.uint8)
    s1, s2 = serial(e, 16)
    return {
        "frequency": frequency(e),
        "block_frequency": block_frequency(e, 128),
        "runs": runs(e),
        "longest_run": longest_run(e),
        "dft": dft(e),
        "linear_complexity": linear_complexity(e, 500),
        "serial_1": s1,
        "serial_2": s2,
        "approximate_entropy": approximate_entropy(e, 10),
        "cusum_forward": cumulative_sums(e),
        "cusum_reverse": cumulative_sums(e, reverse=True),
    }
