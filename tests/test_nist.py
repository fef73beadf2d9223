"""NIST SP 800-22 tests (tests/nist.py): pinned to the worked examples of the
standard, then run on the oracle's output with negative controls (SURVEY
§8(f) f4; the paper's quality claims are P:18 §IV-B).

Pins are the P-values SP 800-22 rev. 1a prints in the "Example" subsection of
each test (§2.x.8), for its short sequences and for its 100-bit example, the
first 100 bits of pi in binary (computed here with Machin's formula, not
typed in); linear complexity is pinned by brute force (the shortest LFSR
that generates a short sequence, found by exhaustive search).
"""
import itertools

import numpy as np
import pytest

import nist as N
import oracle as O

M32 = 1 << 32
ALPHA = 1e-4


def pi_bits(nbits):
    """Leading `nbits` bits of pi = 11.00100100001111110110... (Machin)."""
    prec = nbits + 64

    def atan_inv(x):
        one, s, k = 1 << prec, 0, 0
        t = one // x
        while t:
            s += t // (2 * k + 1) if k % 2 == 0 else -(t // (2 * k + 1))
            t //= x * x
            k += 1
        return s
    v = (4 * (4 * atan_inv(5) - atan_inv(239))) >> (prec - nbits + 2)
    return N.bits_of_string(bin(v)[2:])


@pytest.fixture(scope="module")
def pi100():
    e = pi_bits(100)
    assert e.size == 100 and "".join(map(str, e[:16])) == "1100100100001111"
    return e


def test_sp800_22_short_examples():
    b = N.bits_of_string
    assert N.frequency(b("1011010101")) == pytest.approx(0.527089, abs=1e-6)
    assert N.block_frequency(b("0110011010"), 3) == pytest.approx(0.801252, abs=1e-6)
    assert N.runs(b("1001101011")) == pytest.approx(0.147232, abs=1e-6)
    assert N.approximate_entropy(b("0100110101"), 3) == pytest.approx(0.261961, abs=1e-6)
    p1, p2 = N.serial(b("0011011101"), 3)
    assert p1 == pytest.approx(0.808792, abs=1e-6) and p2 == pytest.approx(0.670320, abs=1e-6)
    assert N.cumulative_sums(b("1011010111")) == pytest.approx(0.4116588, abs=1e-6)
    lr = b("11001100000101010110110001001100111000000000001001001101010100010001001111010110"
           "100000001101011111001100111001101101100010110010")
    assert N.longest_run(lr) == pytest.approx(0.180609, abs=1e-6)
    assert int(N.berlekamp_massey(b("1101011110001")[None, :])[0]) == 4


def test_sp800_22_pi_examples(pi100):
    e = pi100
    assert N.frequency(e) == pytest.approx(0.109599, abs=1e-6)
    assert N.block_frequency(e, 10) == pytest.approx(0.706438, abs=1e-6)
    assert N.runs(e) == pytest.approx(0.500798, abs=1e-6)
    assert N.dft(e) == pytest.approx(0.646355, abs=1e-6)
    assert N.approximate_entropy(e, 2) == pytest.approx(0.235301, abs=1e-6)
    assert N.cumulative_sums(e) == pytest.approx(0.219194, abs=1e-6)
    assert N.cumulative_sums(e, reverse=True) == pytest.approx(0.114866, abs=1e-6)


def test_longest_run_probabilities_exact():
    # M = 8 by counting: longest run <= 1 <=> no two adjacent ones (Fibonacci 55)
    p = N.longest_run_class_probs(8, 1, 4)
    assert np.allclose(p, np.array([55, 94, 59, 48]) / 256.0, rtol=0, atol=1e-15)
    cnt = np.zeros(4)
    for v in range(256):
        s = format(v, "08b")
        cnt[min(max(max(len(r) for r in s.split("0")), 1), 4) - 1] += 1
    assert np.array_equal(cnt, [55, 94, 59, 48])
    for M, (K, lo, hi) in N._LONGEST.items():
        assert N.longest_run_class_probs(M, lo, hi).sum() == pytest.approx(1.0, abs=1e-12)


def _lc_brute(s):
    """Shortest LFSR (length L, any connection polynomial) generating s."""
    n = len(s)
    for L in range(0, n + 1):
        for c in itertools.product((0, 1), repeat=L):
            if all(s[k] == (sum(c[i] * s[k - 1 - i] for i in range(L)) & 1) for k in range(L, n)):
                return L
    return n


def test_berlekamp_massey_equals_brute_force():
    rng = np.random.default_rng(3)
    seqs = rng.integers(0, 2, size=(300, 12), dtype=np.uint8)
    seqs[0] = 0
    seqs[1] = 0
    seqs[1, -1] = 1  # 0...01 has complexity n
    L = N.berlekamp_massey(seqs)
    assert L[0] == 0 and L[1] == 12
    for s, l in zip(seqs, L):
        assert l == _lc_brute(list(s))


def test_berlekamp_massey_recovers_lfsr_length():
    # x^31 + x^3 + 1 is primitive: any nonzero state gives complexity exactly 31
    rng = np.random.default_rng(4)
    rows = []
    for _ in range(8):
        st = list(rng.integers(0, 2, 31))
        if not any(st):
            st[0] = 1
        s = st[:]
        while len(s) < 500:
            s.append(s[-31] ^ s[-28])
        rows.append(s)
    assert list(N.berlekamp_massey(np.array(rows, dtype=np.uint8))) == [31] * 8


@pytest.fixture(scope="module")
def oracle_bits():
    W, D = 2048, 16  # 32768 labels = 2^21 bits
    z = O.bulk(M32, 64, 64, 0x5EED0002, W, 0, W * D)
    return z, W, D


def _run_pass(bits):
    res = N.run(bits)
    return {k: v for k, v in res.items() if v < ALPHA}


def test_oracle_output_passes(oracle_bits):
    z, W, D = oracle_bits
    words = np.ascontiguousarray(z).view(np.uint32)
    bits = N.bits_of_words(words)
    for seq in (bits[:1_000_000], bits[1_000_000:2_000_000]):
        assert not _run_pass(seq)
    # walker-major order: each walker's consecutive draws
    wm = np.ascontiguousarray(z.reshape(D, W).T).reshape(-1).view(np.uint32)
    assert not _run_pass(N.bits_of_words(wm)[:1_000_000])


def test_negative_controls_fail():
    # l = 1 in walker-major order: consecutive outputs are adjacent vertices
    W, D = 64, 256
    z = O.bulk(M32, 1, 64, 0x5EED0002, W, 0, W * D)
    wm = np.ascontiguousarray(z.reshape(D, W).T).reshape(-1).view(np.uint32)
    fails = _run_pass(N.bits_of_words(wm)[:1_000_000])
    assert {"dft", "serial_1", "approximate_entropy"} <= set(fails), fails
    # 32-bit LCG (Numerical Recipes constants): low bits have short periods
    x = np.empty(31250, dtype=np.uint64)
    v = 12345
    for i in range(x.size):
        v = (1664525 * v + 1013904223) & 0xFFFFFFFF
        x[i] = v
    lcg = N.bits_of_words(x.astype(np.uint32))
    assert "dft" in _run_pass(lcg)  # the periodic low bits are spectral lines
    # a biased source: P(1) = 0.505
    rng = np.random.default_rng(9)
    biased = (rng.random(1_000_000) < 0.505).astype(np.uint8)
    assert "frequency" in _run_pass(biased)


def test_host_generator_feed_words_pass():
    # R23 (bit_source 3): the words the host generator feeds (x, y halves of
    # its labels, reseeded per 64-word block) are themselves random-looking
    seed, n_words = 0x5EED0008, 31250
    f = O.lib().or_stream_word32_ggcpu
    w = np.array([f(seed, t, k) for t in range(250) for k in range(125)], dtype=np.uint32)
    assert w.size == n_words
    assert not _run_pass(N.bits_of_words(w))
