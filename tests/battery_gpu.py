"""Crush-scale empirical tests computed with torch on the GPU box (test
infrastructure only).  The paper runs TestU01 (§IV-B,
Table III: SmallCrush 15/15, Crush 14/15, BigCrush 13/15); TestU01 is not
available offline, so this module re-implements 15 statistics of the kinds
Crush/BigCrush are made of, from their textbook laws, as STREAMING tests:
feed() takes a chunk of 64-bit labels (a torch int64 tensor, any device) and
the p-value is computed at the end, so a test can read 2^33 words or more.

  serial_over_t{2,3,4}   overlapping serial test (smultin_MultinomialOver /
                         sknuth_SerialOver): Good's first difference
                         psi2_t - psi2_{t-1} of circular overlapping t-tuples
                         ~ chi2(d^t - d^{t-1})
  collision_b40          (smultin collisions) n balls into 2^40 cells per
                         sample; sum of collisions ~ Poisson(S E[C])
  birthday_spacings_b64  (smarsa_BirthdaySpacings, BigCrush sizes) n = 2^24
                         birthdays in 2^64 days; duplicated spacings ~
                         Poisson(S n^3 / 4k)
  matrix_rank_60, _300   (smarsa_MatrixRank) GF(2) rank law of L x L
  gap                    (sknuth_Gap) geometric gap lengths
  max_of_t               (sknuth_MaxOft) max^t ~ U(0, 1)
  gcd                    (smarsa_GCD) P(gcd = j) -> 6 / (pi^2 j^2)
  hamming_weight         (sstring_HammingWeight2) popcount of 64-bit blocks
                         ~ Binomial(64, 1/2)
  hamming_indep          (sstring_HammingIndep) successive block weights
                         independent
  weight_distrib         (svaria_WeightDistrib) uniforms below 1/4 in groups
                         of 256 ~ Binomial(256, 1/4)
  autocor_d{1,32}        (sstring_AutoCor) XOR of bits d apart ~ Binomial

Word stream: the u32 words of the labels in little-endian order (R12), i.e.
label i gives words 2i (x) and 2i+1 (y).  Uniforms are (word + 0.5) / 2^32.
Nothing here is imported by the product package.
"""
from __future__ import annotations

import math

import numpy as np
import torch
from scipy import stats

MASK32 = 0xFFFFFFFF


def words_of(lab: torch.Tensor) -> torch.Tensor:
    """u32 words (as int64 in [0, 2^32)) of int64 labels, little-endian order."""
    return torch.stack((lab & MASK32, (lab >> 32) & MASK32), dim=1).reshape(-1)


def popcount64(x: torch.Tensor) -> torch.Tensor:
    """Bit count of int64 values (two's complement bits), SWAR."""
    x = x - ((x >> 1) & 0x5555555555555555)
    x = (x & 0x3333333333333333) + ((x >> 2) & 0x3333333333333333)
    x = (x + (x >> 4)) & 0x0F0F0F0F0F0F0F0F
    return ((x * 0x0101010101010101) >> 56) & 0xFF


def chi2_p(counts, probs, min_expected=5.0) -> float:
    """Chi-square p-value, adjacent small cells merged (as tests/battery.py)."""
    counts = np.asarray(counts, dtype=float)
    probs = np.asarray(probs, dtype=float)
    exp = probs * counts.sum()
    oc, ec = [], []
    ao = ae = 0.0
    for o, e in zip(counts, exp):
        ao += o
        ae += e
        if ae >= min_expected:
            oc.append(ao)
            ec.append(ae)
            ao = ae = 0.0
    if ae > 0 and ec:
        oc[-1] += ao
        ec[-1] += ae
    oc, ec = np.array(oc), np.array(ec)
    if oc.size < 2:
        return 1.0
    return float(stats.chi2.sf(((oc - ec) ** 2 / ec).sum(), oc.size - 1))


def poisson_two_sided(x, lam) -> float:
    return float(min(1.0, 2 * min(stats.poisson.cdf(x, lam), stats.poisson.sf(x - 1, lam))))


class SerialOver:
    two_sided = True
    """Overlapping t-tuples of b-bit values (top b bits of each word) on the
    circular sequence; Good (1953): psi2_t - psi2_{t-1} ~ chi2(d^t - d^{t-1}),
    psi2_s = (d^s / n) sum_cells c^2 - n."""

    def __init__(self, t=3, b=8):
        self.t, self.b, self.d = t, b, 1 << b
        self.name = f"serial_over_t{t}_b{b}"
        self.counts = {s: None for s in (t, t - 1)}
        self.head = None    # first t-1 values of the stream
        self.tail = None    # last t-1 values seen
        self.n = 0

    def _tuples(self, v, s):
        idx = torch.zeros(v.numel() - s + 1, dtype=torch.int64, device=v.device)
        for j in range(s):
            idx = idx * self.d + v[j:v.numel() - s + 1 + j]
        return idx

    def _count(self, v, s):
        if v.numel() < s:
            return
        c = torch.bincount(self._tuples(v, s), minlength=self.d ** s)
        self.counts[s] = c if self.counts[s] is None else self.counts[s] + c

    def feed(self, lab):
        v = words_of(lab) >> (32 - self.b)
        if self.head is None:
            self.head = v[: self.t - 1].clone()
        ext = v if self.tail is None else torch.cat((self.tail, v))
        # every tuple that ENDS in this chunk: start at ext index >= len(tail) - (s-1)
        off = 0 if self.tail is None else self.tail.numel()
        for s in (self.t, self.t - 1):
            self._count(ext[max(0, off - (s - 1)):], s)
        self.tail = ext[-(self.t - 1):].clone()
        self.n += v.numel()

    def pvalue(self):
        # wrap-around tuples of the circular sequence
        ext = torch.cat((self.tail, self.head))
        for s in (self.t, self.t - 1):
            k = self.t - 1          # len(tail)
            self._count(ext[k - (s - 1): k + (s - 1)], s)
        n = self.n
        psi = {}
        for s in (self.t, self.t - 1):
            c = self.counts[s].to(torch.float64)
            assert int(self.counts[s].sum()) == n
            psi[s] = (self.d ** s / n) * float((c * c).sum()) - n
        stat = psi[self.t] - psi[self.t - 1]
        df = self.d ** self.t - self.d ** (self.t - 1)
        return float(2 * min(stats.chi2.sf(stat, df), stats.chi2.cdf(stat, df)))


class Collision:
    two_sided = True
    """n labels per sample hashed to their top `bits` bits (k = 2^bits cells);
    collisions C = n - distinct cells; E[C] = n - k + k (1 - 1/k)^n; the sum
    over samples is Poisson for n^2/k small relative to n."""

    def __init__(self, bits=40, n=1 << 24):
        self.bits, self.n = bits, n
        self.name = f"collision_b{bits}"
        self.buf = []
        self.have = 0
        self.C = 0
        self.S = 0

    def _sample(self, keys):
        s = torch.sort(keys).values
        self.C += int((s[1:] == s[:-1]).sum())
        self.S += 1

    def feed(self, lab):
        keys = (lab >> (64 - self.bits)) & ((1 << self.bits) - 1)
        self.buf.append(keys)
        self.have += keys.numel()
        if self.have >= self.n:
            allk = torch.cat(self.buf)
            m = allk.numel() // self.n
            for i in range(m):
                self._sample(allk[i * self.n:(i + 1) * self.n])
            rest = allk[m * self.n:]
            self.buf = [rest] if rest.numel() else []
            self.have = rest.numel()

    def pvalue(self):
        k = float(2 ** self.bits)
        e = self.n - k * (-math.expm1(self.n * math.log1p(-1.0 / k)))
        return poisson_two_sided(self.C, self.S * e)


class BirthdaySpacings(Collision):
    """Marsaglia's birthday spacings: n birthdays = top `bits` bits of n
    labels in k = 2^bits days (bits = 64: the full label, BigCrush sizes);
    sort, the n circular spacings, Y = repeated spacings (sorted adjacent
    equal); Y ~ Poisson(n^3 / 4k) per sample."""

    def __init__(self, n=1 << 24, bits=64):
        super().__init__(bits=bits, n=n)
        self.name = f"birthday_spacings_b{bits}"

    def _sample(self, lab):
        if self.bits == 64:
            # signed order is a rotation of the unsigned circle; differences
            # wrap modulo 2^64 in two's complement
            s = torch.sort(lab).values
            sp = torch.cat((s[1:] - s[:-1], s[:1] - s[-1:]))
        else:
            s = torch.sort((lab >> (64 - self.bits)) & ((1 << self.bits) - 1)).values
            sp = torch.cat((s[1:] - s[:-1], s[:1] + (1 << self.bits) - s[-1:]))
        sp = torch.sort(sp).values
        self.C += int((sp[1:] == sp[:-1]).sum())
        self.S += 1

    def feed(self, lab):
        self.buf.append(lab)
        self.have += lab.numel()
        if self.have >= self.n:
            allk = torch.cat(self.buf)
            m = allk.numel() // self.n
            for i in range(m):
                self._sample(allk[i * self.n:(i + 1) * self.n])
            rest = allk[m * self.n:]
            self.buf = [rest] if rest.numel() else []
            self.have = rest.numel()

    def pvalue(self):
        lam = float(self.n) ** 3 / (4.0 * 2.0 ** self.bits)
        return poisson_two_sided(self.C, self.S * lam)


def gf2_rank_probs(L):
    """P(rank = r) of an L x L uniform binary matrix, r = 0..L:
    2^(r(2L - r) - L^2) prod_{i<r} (1 - 2^(i-L))^2 / (1 - 2^(i-r))."""
    out = []
    for r in range(L + 1):
        lv = (r * (2 * L - r) - L * L) * math.log(2.0)
        for i in range(r):
            lv += 2 * math.log1p(-2.0 ** (i - L)) - math.log1p(-2.0 ** (i - r))
        out.append(math.exp(lv))
    return out


def gf2_ranks(rows: torch.Tensor, L: int) -> torch.Tensor:
    """Ranks over GF(2) of B matrices: rows [B, L, words] int64, bit c of a
    row = bit (c % 64) of word c // 64, columns c < L."""
    B = rows.shape[0]
    dev = rows.device
    rows = rows.clone()
    used = torch.zeros(B, L, dtype=torch.bool, device=dev)
    rank = torch.zeros(B, dtype=torch.int64, device=dev)
    ar = torch.arange(B, device=dev)
    for c in range(L):
        w, sh = divmod(c, 64)
        bit = ((rows[:, :, w] >> sh) & 1).bool()
        cand = bit & ~used
        has = cand.any(dim=1)
        piv = cand.to(torch.int8).argmax(dim=1)
        prow = rows[ar, piv]                                  # [B, words]
        elim = bit & has[:, None]
        elim[ar, piv] = False
        rows = torch.where(elim[:, :, None], rows ^ prow[:, None, :], rows)
        used[ar, piv] |= has
        rank += has.to(torch.int64)
    return rank


class MatrixRank:
    """smarsa_MatrixRank: L x L matrices; a row is L consecutive bits of the
    label stream (one label per row for L <= 64, ceil(L/64) labels else);
    chi-square over ranks L, L-1, L-2, <= L-3.  max_matrices bounds the work
    (the 300 x 300 elimination is O(L^2) vector steps per batch)."""

    def __init__(self, L=60, batch=1 << 18, max_matrices=None):
        self.L, self.batch, self.maxm = L, batch, max_matrices
        self.wpr = (L + 63) // 64           # labels (64-bit words) per row
        self.per = self.L * self.wpr         # labels per matrix
        self.name = f"matrix_rank_{L}"
        self.hist = np.zeros(4, dtype=np.int64)
        self.buf, self.have = [], 0

    def _run(self, lab):
        m = lab.numel() // self.per
        if self.maxm is not None:
            m = min(m, self.maxm - int(self.hist.sum()))
        if m <= 0:
            return
        rows = lab[: m * self.per].reshape(m, self.L, self.wpr).clone()
        last = self.L - 64 * (self.wpr - 1)   # bits used in the last word of a row
        if last < 64:
            rows[:, :, -1] &= (1 << last) - 1
        for i in range(0, m, self.batch):
            r = gf2_ranks(rows[i:i + self.batch], self.L)
            d = (self.L - r).clamp(max=3)
            self.hist += np.bincount(d.cpu().numpy(), minlength=4)[:4]

    def feed(self, lab):
        if self.maxm is not None and self.hist.sum() >= self.maxm:
            return
        self.buf.append(lab)
        self.have += lab.numel()
        if self.have >= self.per * 1024:
            allk = torch.cat(self.buf)
            m = allk.numel() // self.per
            self._run(allk[: m * self.per])
            rest = allk[m * self.per:]
            self.buf, self.have = ([rest] if rest.numel() else []), rest.numel()

    def pvalue(self):
        if self.buf:
            self._run(torch.cat(self.buf))
            self.buf = []
        p = gf2_rank_probs(self.L)
        probs = [p[self.L], p[self.L - 1], p[self.L - 2], sum(p[: self.L - 2])]
        return chi2_p(self.hist, probs, min_expected=1.0)


class Gap:
    """sknuth_Gap: U in [alpha, beta) marks a hit; gap g = non-hits between
    hits ~ geometric, P(g = k) = p (1-p)^k, categories 0..t-1 and >= t."""

    def __init__(self, alpha=0.0, beta=1 / 16, t=64):
        self.a, self.b, self.t = int(alpha * 2 ** 32), int(beta * 2 ** 32), t
        self.p = beta - alpha
        self.name = "gap"
        self.hist = None
        self.last = None
        self.pos = 0

    def feed(self, lab):
        w = words_of(lab)
        hit = torch.nonzero((w >= self.a) & (w < self.b)).flatten() + self.pos
        if self.last is not None:
            hit = torch.cat((torch.tensor([self.last], device=hit.device), hit))
        if hit.numel() >= 2:
            g = (hit[1:] - hit[:-1] - 1).clamp(max=self.t)
            h = torch.bincount(g, minlength=self.t + 1).cpu().numpy()
            self.hist = h if self.hist is None else self.hist + h
        if hit.numel():
            self.last = int(hit[-1])
        self.pos += w.numel()

    def pvalue(self):
        k = np.arange(self.t)
        probs = list(self.p * (1 - self.p) ** k) + [(1 - self.p) ** self.t]
        return chi2_p(self.hist, probs)


class MaxOfT:
    """sknuth_MaxOft: V = max of t uniforms, V^t ~ U(0,1), chi-square on
    `cells` equiprobable cells."""

    def __init__(self, t=8, cells=1024):
        self.t, self.cells = t, cells
        self.name = "max_of_t"
        self.hist = np.zeros(cells, dtype=np.int64)
        self.carry = None

    def feed(self, lab):
        w = words_of(lab)
        if self.carry is not None:
            w = torch.cat((self.carry, w))
        m = w.numel() // self.t
        self.carry = w[m * self.t:].clone()
        v = (w[: m * self.t].reshape(m, self.t).max(dim=1).values.to(torch.float64) + 0.5) / 2.0 ** 32
        c = (v.pow(self.t) * self.cells).to(torch.int64).clamp(max=self.cells - 1)
        self.hist += torch.bincount(c, minlength=self.cells).cpu().numpy()

    def pvalue(self):
        return chi2_p(self.hist, [1.0 / self.cells] * self.cells)


class GCD:
    """smarsa_GCD (Marsaglia & Tsang 2002): gcd of successive word pairs
    (zero words skipped), P(gcd = j) -> 6 / (pi^2 j^2), j >= jmax pooled."""

    def __init__(self, jmax=64):
        self.jmax = jmax
        self.name = "gcd"
        self.hist = np.zeros(jmax + 1, dtype=np.int64)

    def feed(self, lab):
        w = words_of(lab).reshape(-1, 2)
        w = w[(w[:, 0] > 0) & (w[:, 1] > 0)]
        g = torch.gcd(w[:, 0], w[:, 1]).clamp(max=self.jmax)
        self.hist += torch.bincount(g, minlength=self.jmax + 1).cpu().numpy()

    def pvalue(self):
        p = [6.0 / (math.pi ** 2 * j * j) for j in range(1, self.jmax)]
        return chi2_p(self.hist[1:], p + [1.0 - sum(p)])


class HammingWeight:
    """Popcount of each 64-bit label ~ Binomial(64, 1/2)."""

    def __init__(self):
        self.name = "hamming_weight"
        self.hist = np.zeros(65, dtype=np.int64)

    def feed(self, lab):
        self.hist += torch.bincount(popcount64(lab), minlength=65).cpu().numpy()

    def pvalue(self):
        return chi2_p(self.hist, stats.binom.pmf(np.arange(65), 64, 0.5))


class HammingIndep:
    """sstring_HammingIndep: weights of disjoint successive label pairs,
    binned (<= 28, 29..35 individually, >= 36), against the product of the
    Binomial(64, 1/2) marginals."""

    EDGES = (28, 29, 30, 31, 32, 33, 34, 35)

    def __init__(self):
        self.name = "hamming_indep"
        nb = len(self.EDGES) + 1
        self.nb = nb
        self.hist = np.zeros(nb * nb, dtype=np.int64)
        self.edges = None

    def feed(self, lab):
        w = popcount64(lab[: lab.numel() // 2 * 2])
        if self.edges is None:
            self.edges = torch.tensor(self.EDGES, device=lab.device)
        b = torch.bucketize(w, self.edges, right=False)   # 0: <= 28 ... nb-1: >= 36
        cell = b[0::2] * self.nb + b[1::2]
        self.hist += torch.bincount(cell, minlength=self.nb * self.nb).cpu().numpy()

    def pvalue(self):
        e = self.EDGES
        pm = np.array([stats.binom.cdf(e[0], 64, 0.5)] +
                      [stats.binom.pmf(c, 64, 0.5) for c in e[1:]] +
                      [stats.binom.sf(e[-1], 64, 0.5)])
        return chi2_p(self.hist, np.outer(pm, pm).ravel())


class AutoCor:
    two_sided = True
    """sstring_AutoCor: over the bit stream (words in order, each word's bits
    least significant first), A = sum_i b_i XOR b_{i+d} ~ Binomial(N, 1/2);
    d = 1 (within and across words) or d = 32 (word i vs word i+1)."""

    def __init__(self, d=1):
        assert d in (1, 32)
        self.d = d
        self.name = f"autocor_d{d}"
        self.A = 0
        self.N = 0
        self.prev = None  # last word of the previous chunk

    def feed(self, lab):
        w = words_of(lab)
        if self.prev is not None:
            w = torch.cat((self.prev, w))
        nxt = w[1:]
        cur = w[:-1]
        if self.d == 32:
            x = cur ^ nxt
        else:  # bit i vs bit i+1: word shifted right by one, top bit from the next word
            x = (cur ^ ((cur >> 1) | ((nxt & 1) << 31))) & MASK32
        self.A += int(popcount64(x).sum())
        self.N += 32 * cur.numel()
        self.prev = w[-1:].clone()

    def pvalue(self):
        z = (self.A - self.N / 2) / math.sqrt(self.N / 4)
        return float(2 * stats.norm.sf(abs(z)))


class WeightDistrib:
    """svaria_WeightDistrib: number of uniforms below beta in groups of k
    ~ Binomial(k, beta)."""

    def __init__(self, k=256, beta=0.25):
        self.k, self.beta = k, beta
        self.thr = int(beta * 2 ** 32)
        self.name = "weight_distrib"
        self.hist = np.zeros(k + 1, dtype=np.int64)
        self.carry = None

    def feed(self, lab):
        w = words_of(lab)
        if self.carry is not None:
            w = torch.cat((self.carry, w))
        m = w.numel() // self.k
        self.carry = w[m * self.k:].clone()
        c = (w[: m * self.k].reshape(m, self.k) < self.thr).sum(dim=1)
        self.hist += torch.bincount(c, minlength=self.k + 1).cpu().numpy()

    def pvalue(self):
        return chi2_p(self.hist, stats.binom.pmf(np.arange(self.k + 1), self.k, self.beta))


def crush_scale_tests(rank300_matrices=1 << 15, samples_n=1 << 24):
    """The 15 streaming statistics, fresh state."""
    return [SerialOver(2, 12), SerialOver(3, 8), SerialOver(4, 6),
            Collision(40, samples_n), BirthdaySpacings(samples_n),
            MatrixRank(60), MatrixRank(300, batch=1 << 12, max_matrices=rank300_matrices),
            Gap(), MaxOfT(), GCD(), HammingWeight(), HammingIndep(), WeightDistrib(),
            AutoCor(1), AutoCor(32)]


def verdict(test, p, lo=1e-4):
    """TestU01-style reading: a one-sided (chi-square right tail) p-value
    fails outside [lo, 1 - lo] (a fit too good is as suspect as a bad one);
    a two-sided p-value fails below lo.  lo = 1e-4 here; TestU01 lists p
    outside [0.001, 0.999] and calls < 1e-10 a clear failure."""
    if getattr(test, "two_sided", False):
        return "pass" if p >= lo else "fail"
    return "pass" if lo <= p <= 1 - lo else "fail"
