"""Pins for the CPU oracle's generator core (no GPU).

Each test fixes the oracle against something other than itself:
published SplitMix64 outputs, hand-worked neighbour lists from PAPER.md:14
§III-A, an independent computation, exhaustive graph
invariants, the closed-form parity-chain decay, brute-force mixing at the
spectral rate, and the Z/2^32 -> Z/2^k ring homomorphism.  A dropped term,
a wrong sign/index or a transposed coordinate fails at least one of them.
"""
import numpy as np
import pytest

import oracle as O
from conftest import read_golden

M32 = 1 << 32


# ---------------------------------------------------------------- P1 vectors
def test_splitmix64_published_outputs():
    for row in read_golden("splitmix64_seed0.txt"):
        kind, t, c, val = row[0], int(row[1]), int(row[2]), int(row[3], 16)
        if kind == "word64":
            assert O.stream_word64(0, t, c) == val
        else:
            assert O.stream_word32(0, t, c) == val


def test_single_steps_hand_worked():
    for row in read_golden("gg_single_step.txt"):
        if row[0] == "seq":
            m, x, y = int(row[1]), int(row[2], 16), int(row[3], 16)
            bs = [int(b) for b in row[4].split(",")]
            labels = [int(v, 16) for v in row[5].split(",")]
            for b, lab in zip(bs, labels):
                x, y = O.walk(m, x, y, np.array([b], np.uint32), 1)
                assert O.label(m, x, y) == lab
        else:
            m, x, y, b, nx, ny = (int(v) for v in row)
            assert O.walk(m, x, y, np.array([b], np.uint32), 1) == (nx, ny)


def test_full_generator_vectors():
    for row in read_golden("gg_full_generator.txt"):
        if row[0] == "bulk":
            m, W, g0 = int(row[1]), int(row[2]), int(row[3])
            want = [int(v) for v in row[4].split(",")]
            got = O.bulk(m, 64, 64, 0, W, g0, len(want))
            assert list(map(int, got)) == want
            continue
        m, t, j, val = int(row[0]), int(row[1]), int(row[2]), int(row[3], 0)
        if j < 0:
            x, y = O.walker_init(m, 64, 0, t)
            assert O.label(m, x, y) == val
        else:
            assert int(O.walker_draws(m, 64, 64, 0, t, j, 1)[0]) == val


def test_start_vertex_uses_first_64_bits():
    # Alg.1: "To select the starting position, we need 64 random bits";
    # R7: x = word 0, y = word 1 (mod m).  With l0 = 0 the walk is empty.
    for t in (0, 5, 77):
        x, y = O.walker_init(M32, 0, 123, t)
        assert x == O.stream_word32(123, t, 0) and y == O.stream_word32(123, t, 1)
        x8, y8 = O.walker_init(256, 0, 123, t)
        assert (x8, y8) == (x % 256, y % 256)


# ------------------------------------------------------------- R3 bit order
def test_bit_order_little_endian_fields():
    # A single set bit at position p of the record is seen by step p // 3 as
    # the value 1 << (p % 3) and by no other step (R3), including the fields
    # that straddle 32-bit words (steps 10, 21, 42, 53 of a 64-step walk).
    for p in range(192):
        rec = np.zeros(6, np.uint32)
        rec[p // 32] = np.uint32(1 << (p % 32))
        vals = [O.bits3(rec, i) for i in range(64)]
        want = [0] * 64
        want[p // 3] = 1 << (p % 3)
        assert vals == want, p
    assert O.words_per_walk(64) == 6 and O.words_per_walk(1) == 1 and O.words_per_walk(11) == 2


def test_walk_value7_is_stay_and_reads_fields_in_order():
    # R4: b = 7 selects sigma_0.  An all-ones record never moves.
    ones = np.full(6, 0xFFFFFFFF, np.uint32)
    assert O.walk(M32, 123, 456, ones, 64) == (123, 456)
    # A record whose only nonzero field is step 63 = b:1 moves only at the end.
    rec = np.zeros(6, np.uint32)
    rec[5] = np.uint32(1 << 29)  # bit 189 = field 63, value 1
    assert O.walk(M32, 3, 4, rec, 64) == (3, 2 * 3 + 4)
    assert O.walk(M32, 3, 4, rec, 63) == (3, 4)


# ------------------------------------------------- P2 bijectivity/regularity
@pytest.mark.parametrize("m", [2, 3, 4, 5, 7, 8, 16, 31, 32, 64])
def test_each_sigma_is_bijection_and_graph_is_7_regular(m):
    xs, ys = np.meshgrid(np.arange(m, dtype=np.uint64), np.arange(m, dtype=np.uint64), indexing="ij")
    xs, ys = xs.ravel(), ys.ravel()
    indeg = np.zeros(m * m, np.int64)
    for k in range(7):
        nx, ny = O.sigma(m, k, xs, ys)
        assert nx.max() < m and ny.max() < m
        ids = (nx + np.uint64(m) * ny).astype(np.int64)
        assert np.unique(ids).size == m * m, (m, k)
        indeg += np.bincount(ids, minlength=m * m)
    # every vertex has out-degree 7 (by construction) and in-degree 7
    assert np.all(indeg == 7)


def _transition_from_walk(m):
    """Row-stochastic transition over Z_m^2 built from the oracle's walk with
    every 3-bit value b (each with probability 1/8): exercises bits3, the
    b mod 7 rule and sigma together."""
    n = m * m
    Pm = np.zeros((n, n))
    for x in range(m):
        for y in range(m):
            for b in range(8):
                nx, ny = O.walk(m, x, y, np.array([b], np.uint32), 1)
                Pm[x + m * y, nx + m * ny] += 1.0 / 8
    return Pm


@pytest.mark.parametrize("m", [3, 4, 8])
def test_uniform_is_stationary_doubly_stochastic(m):
    # P3: each sigma_k is a bijection, so P is doubly stochastic and the
    # uniform distribution is stationary: every output's marginal is uniform.
    Pm = _transition_from_walk(m)
    assert np.allclose(Pm.sum(axis=1), 1.0) and np.allclose(Pm.sum(axis=0), 1.0)
    u = np.full(m * m, 1.0 / (m * m))
    assert np.allclose(u @ Pm, u, atol=1e-15)


@pytest.mark.parametrize("m", [4, 8])
def test_parity_chain_closed_form(m):
    # P4: x mod 2 flips only on sigma_5 (x+2y+1), y mod 2 only on sigma_2
    # (2x+y+1), each with probability 1/8, so from (0,0)
    #   Pr[x_t odd] = Pr[y_t odd] = (1 - (3/4)^t) / 2.
    Pm = _transition_from_walk(m)
    d = np.zeros(m * m)
    d[0] = 1.0
    ids = np.arange(m * m)
    xodd, yodd = (ids % m) % 2 == 1, (ids // m) % 2 == 1
    for t in range(1, 25):
        d = d @ Pm
        want = (1 - 0.75 ** t) / 2
        assert abs(d[xodd].sum() - want) < 1e-12
        assert abs(d[yodd].sum() - want) < 1e-12
    # and the second-largest eigenvalue modulus is 3/4
    ev = np.sort(np.abs(np.linalg.eigvals(Pm)))[::-1]
    assert abs(ev[0] - 1) < 1e-9 and abs(ev[1] - 0.75) < 1e-9


def _tv_curve(m, start, tmax):
    n = m * m
    xs, ys = np.meshgrid(np.arange(m, dtype=np.uint64), np.arange(m, dtype=np.uint64), indexing="ij")
    src = (xs + np.uint64(m) * ys).ravel().astype(np.int64)
    xs, ys = xs.ravel(), ys.ravel()
    dst = []
    for b in range(8):
        # k = b mod 7 (R4); sigma from the oracle
        nx, ny = O.sigma(m, b % 7, xs, ys)
        d_ = np.empty(n, np.int64)
        d_[src] = (nx + np.uint64(m) * ny).astype(np.int64)
        dst.append(d_)
    d = np.zeros(n)
    d[start] = 1.0
    tv = []
    for t in range(1, tmax + 1):
        nd = np.zeros(n)
        for b in range(8):
            nd += np.bincount(dst[b], weights=d, minlength=n)
        d = nd / 8
        tv.append(0.5 * np.abs(d - 1.0 / n).sum())
    return np.array(tv)


def test_bruteforce_mixing_m256():
    # P5/P6: "random walks on expander graphs have a rapid mixing property"
    # (§III-A).  Brute-force TV distance from (0,0) on m = 2^8 (65 536
    # states) vs the independent SURVEY §A.1 numbers, and the decay rate
    # approaching the closed-form |lambda_2| = 3/4.
    tv = _tv_curve(256, 0, 96)
    assert abs(tv[32 - 1] / 5.27e-4 - 1) < 0.01
    assert abs(tv[64 - 1] / 6.74e-9 - 1) < 0.01
    assert abs(tv[96 - 1] / 5.25e-13 - 1) < 0.02
    rate = (tv[96 - 1] / tv[64 - 1]) ** (1 / 32)
    assert 0.73 < rate < 0.76
    assert np.all(np.diff(tv[8:]) < 0)  # monotone decay


# ----------------------------------------------- P15 ring homomorphism
@pytest.mark.parametrize("k", [1, 2, 8, 13, 16, 31])
def test_power_of_two_m_is_reduction_of_m32(k):
    # Z/2^32 -> Z/2^k is a ring homomorphism, so with identical bits the
    # m = 2^k walk equals the m = 2^32 walk reduced per coordinate.
    mk = 1 << k
    for t in (0, 1, 1023, 99991):
        full = O.walker_draws(M32, 64, 64, 7, t, 0, 4)
        small = O.walker_draws(mk, 64, 64, 7, t, 0, 4)
        fx, fy = full & np.uint64(0xFFFFFFFF), full >> np.uint64(32)
        want = (fx % np.uint64(mk)) + np.uint64(mk) * (fy % np.uint64(mk))
        assert np.array_equal(small, want)


def test_bulk_order_matches_per_walker_draws():
    # R11: Z[g] = label(walker g mod W, draw g div W), and a fill can start
    # at any offset g0 (chunked fills continue the same sequence).
    W = 8
    z = O.bulk(256, 64, 64, 5, W, 0, 50)
    for t in range(W):
        d = O.walker_draws(256, 64, 64, 5, t, 0, 7)
        for j in range(7):
            g = j * W + t
            if g < 50:
                assert z[g] == d[j]
    assert np.array_equal(O.bulk(256, 64, 64, 5, W, 13, 20), z[13:33])


def test_general_l_uses_ceil_3l_over_32_words():
    # Alg.2 with l = 1 (one 3-bit field per draw in its own word) and l = 11
    # (33 bits -> 2 words): the draw record of walker t, draw j starts at word
    # 2 + ceil(3*l0/32) + ceil(3*l/32)*j.
    seed, t = 9, 3
    for l in (1, 11, 64, 100):
        x, y = O.walker_init(M32, 64, seed, t)
        R = O.words_per_walk(l)
        for j in range(3):
            rec = np.array([O.stream_word32(seed, t, 2 + 6 + R * j + r) for r in range(R)], np.uint32)
            x, y = O.walk(M32, x, y, rec, l)
            assert int(O.walker_draws(M32, l, 64, seed, t, j, 1)[0]) == O.label(M32, x, y)


# ------------------------------------------- f1: bipartite variant (σ / σ⁻¹)
@pytest.mark.parametrize("m", [2, 5, 8, 16])
def test_inverse_maps_exhaustive(m):
    # sigma_k^{-1} undoes sigma_k on every vertex (the neighbours in X of a
    # vertex of Y are its preimages), for all k
    for k in range(7):
        for x in range(m):
            for y in range(m):
                nx, ny = O.sigma(m, k, np.array([x], np.uint64), np.array([y], np.uint64))
                assert O.sigma_inv(m, k, int(nx[0]), int(ny[0])) == (x, y)


def test_bipartite_walk_parity_chain_and_alternation():
    # The bipartite walk alternates sigma (even steps) and sigma^{-1} (odd);
    # x mod 2 still flips only on k = 5 (x +- 2y +- 1), so the closed form
    # (1 - (3/4)^t)/2 of P4 holds, and the 2-step chain is doubly stochastic.
    m = 8
    n = m * m
    Pf = np.zeros((n, n))
    Pb = np.zeros((n, n))
    for x in range(m):
        for y in range(m):
            for b in range(8):
                rec = np.array([b], np.uint32)
                xs, ys = np.array([x], np.uint64), np.array([y], np.uint64)
                O.lib().or_walk_bipartite(m, O._ptr(xs), O._ptr(ys), O._ptr(rec), 1, 0)
                Pf[x + m * y, int(xs[0]) + m * int(ys[0])] += 1 / 8
                xs, ys = np.array([x], np.uint64), np.array([y], np.uint64)
                O.lib().or_walk_bipartite(m, O._ptr(xs), O._ptr(ys), O._ptr(rec), 1, 1)
                Pb[x + m * y, int(xs[0]) + m * int(ys[0])] += 1 / 8
    assert np.allclose(Pf.sum(0), 1) and np.allclose(Pb.sum(0), 1)
    d = np.zeros(n)
    d[0] = 1
    xodd = (np.arange(n) % m) % 2 == 1
    for t in range(1, 21):
        d = d @ (Pf if t % 2 == 1 else Pb)
        assert abs(d[xodd].sum() - (1 - 0.75 ** t) / 2) < 1e-12
    # variant 1 differs from variant 0 (odd steps go backwards)
    assert not np.array_equal(O.bulk_v(256, 64, 64, 1, 3, 16, 0, 64), O.bulk_v(256, 64, 64, 0, 3, 16, 0, 64))
    assert np.array_equal(O.bulk_v(256, 64, 64, 0, 3, 16, 0, 64), O.bulk(256, 64, 64, 3, 16, 0, 64))
