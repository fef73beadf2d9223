"""Pins for the Crush-scale streaming battery (tests/battery_gpu.py; SURVEY
§8(f) f4, §IV-B Table III), on CPU tensors:
  * the laws: GF(2) rank probabilities by enumeration of all 3x3 and 4x4
    matrices; collision expectation by enumeration; popcount by Python;
  * the streaming bookkeeping: chunked feeding equals one feed, and the
    circular overlapping tuple counts equal a direct count;
  * null calibration: on numpy PCG64 output every statistic's p-values are
    uniform over replicates (KS), at small sizes;
  * power: a 32-bit LCG's low-bit words and a sequence with serial
    correlation fail the tests they should fail.
"""
import itertools
import math

import numpy as np
import pytest
import torch
from scipy import stats

import battery_gpu as G


def pcg_labels(n, seed):
    rng = np.random.default_rng(seed)
    return torch.from_numpy(rng.integers(0, 2 ** 63, n, dtype=np.int64) ^
                            (rng.integers(0, 2, n, dtype=np.int64) << 63))


def test_popcount64():
    rng = np.random.default_rng(1)
    x = rng.integers(-2 ** 63, 2 ** 63 - 1, 4096, dtype=np.int64)
    got = G.popcount64(torch.from_numpy(x)).numpy()
    want = [bin(int(v) & (2 ** 64 - 1)).count("1") for v in x]
    assert list(got) == want


@pytest.mark.parametrize("L", [3, 4])
def test_gf2_rank_law_by_enumeration(L):
    counts = np.zeros(L + 1)
    rows = []
    for bits in range(1 << (L * L)):
        rows.append([(bits >> (L * i)) & ((1 << L) - 1) for i in range(L)])
    r = G.gf2_ranks(torch.tensor(rows, dtype=torch.int64)[:, :, None], L).numpy()
    counts = np.bincount(r, minlength=L + 1) / (1 << (L * L))
    assert np.allclose(counts, G.gf2_rank_probs(L), rtol=0, atol=1e-15)


def test_gf2_ranks_multiword_against_row_reduction():
    # 70 x 70 matrices (two words per row) vs a plain Python elimination
    rng = np.random.default_rng(2)
    B, L = 24, 70
    m = rng.integers(0, 2, (B, L, L))
    m[:8, 5] = m[:8, 3] ^ m[:8, 9]       # force rank deficiency in some
    words = np.zeros((B, L, 2), dtype=np.int64)
    for c in range(L):
        words[:, :, c // 64] |= m[:, :, c].astype(np.int64) << (c % 64)
    got = G.gf2_ranks(torch.from_numpy(words), L).numpy()
    for b in range(B):
        rows = [int("".join(map(str, m[b, i, ::-1])), 2) for i in range(L)]
        rank = 0
        for c in range(L):
            piv = next((i for i in range(rank, L) if rows[i] >> c & 1), None)
            if piv is None:
                continue
            rows[rank], rows[piv] = rows[piv], rows[rank]
            for i in range(L):
                if i != rank and rows[i] >> c & 1:
                    rows[i] ^= rows[rank]
            rank += 1
        assert got[b] == rank


def test_collision_expectation_by_enumeration():
    k, n = 5, 4
    tot = 0
    for cells in itertools.product(range(k), repeat=n):
        tot += n - len(set(cells))
    want = tot / k ** n
    e = n - k * (-math.expm1(n * math.log1p(-1.0 / k)))
    assert e == pytest.approx(want, rel=1e-12)


def test_serial_over_circular_counts_and_chunking():
    lab = pcg_labels(999, 3)
    a = G.SerialOver(3, 2)
    a.feed(lab)
    b = G.SerialOver(3, 2)
    for i in range(0, 999, 100):
        b.feed(lab[i:i + 100])
    pa, pb = a.pvalue(), b.pvalue()
    assert pa == pb
    for s in (3, 2):
        assert torch.equal(a.counts[s], b.counts[s])
    v = (G.words_of(lab) >> 30).tolist()
    n = len(v)
    for s in (3, 2):
        direct = np.zeros(4 ** s, dtype=np.int64)
        for i in range(n):
            idx = 0
            for j in range(s):
                idx = idx * 4 + v[(i + j) % n]
            direct[idx] += 1
        assert np.array_equal(a.counts[s].numpy(), direct)


def _run(test, lab, chunk=1 << 14):
    for i in range(0, lab.numel(), chunk):
        test.feed(lab[i:i + chunk])
    return test.pvalue()


SMALL = [lambda: G.SerialOver(2, 6), lambda: G.SerialOver(3, 4), lambda: G.Collision(24, 1 << 12),
         lambda: G.BirthdaySpacings(1 << 10, bits=32), lambda: G.MatrixRank(60, batch=256),
         lambda: G.Gap(t=32), lambda: G.MaxOfT(8, 64), lambda: G.GCD(24),
         lambda: G.HammingWeight(), lambda: G.HammingIndep(), lambda: G.WeightDistrib(64),
         lambda: G.AutoCor(1), lambda: G.AutoCor(32)]


@pytest.mark.parametrize("make", SMALL)
def test_null_calibration_pcg64(make):
    """p-values of each statistic on good random bits are uniform: KS over
    replicates (and never an extreme value)."""
    ps = [_run(make(), pcg_labels(1 << 15, 100 + r)) for r in range(24)]
    t = make()
    assert all(G.verdict(t, p) == "pass" for p in ps), (t.name, ps)
    if t.name.startswith(("collision", "birthday")):  # discrete Poisson p-values
        return
    assert stats.kstest(ps, "uniform").pvalue > 1e-3, (t.name, ps)


def test_power_lcg_and_correlated_sequences():
    # 32-bit LCG (Numerical Recipes' a, c), both words of a label are
    # successive outputs: low bits have short periods
    n = 1 << 16
    x = np.empty(2 * n, dtype=np.uint64)
    s = np.uint64(12345)
    a, c, m = np.uint64(1664525), np.uint64(1013904223), np.uint64(0xFFFFFFFF)
    for i in range(2 * n):
        s = (a * s + c) & m
        x[i] = s
    lab = torch.from_numpy((x[0::2] | (x[1::2] << np.uint64(32))).view(np.int64))
    for make in (lambda: G.AutoCor(32), lambda: G.MatrixRank(60, batch=256), lambda: G.GCD(24),
                 lambda: G.HammingWeight(), lambda: G.HammingIndep()):
        assert _run(make(), lab) < 1e-10
    # bit-level lag-1 correlation: every odd bit copies the even bit below it
    r = pcg_labels(n, 9)
    odd = -0x5555555555555556  # 0xAAAA...AAAA as int64
    b = (r & ~odd) | ((r << 1) & odd)
    assert _run(G.AutoCor(1), b) < 1e-10
    # serial correlation: the x word of every label repeats the top byte of its y word
    w = pcg_labels(n, 7)
    w2 = (w & ~(0xFF << 24)) | (((w >> 56) & 0xFF) << 24)
    assert _run(G.SerialOver(2, 8), w2) < 1e-10
