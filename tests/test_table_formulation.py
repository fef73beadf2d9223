"""Host-side check of the composed-step ("table") walk (gg_fill64t_tma_kernel,
csrc/gg_walk.cu), no GPU.

Four consecutive Gabber-Galil steps (§III-A; k = field mod 7, R4)
compose to one affine map x' = a x + b y + e, y' = c x + d y + f over Z/2^32;
the kernel looks the six coefficients up in a 4096-entry table indexed by the
group's 12 record bits (R3) and unpacks them from one 32-bit word
(5-5-5-5-6-6 bits).  This test re-expresses that recipe in Python -- the
composition, the packing, the 12-bit group extraction across word boundaries
and the wrapped arithmetic -- and checks it against the oracle's plain
step-by-step walk, plus the coefficient bounds the packing relies on.
"""
import itertools

import numpy as np

import oracle as O

M = 0xFFFFFFFF


def compose4(p):
    a, b, e, c, d, f = 1, 0, 0, 0, 1, 0
    for i in range(4):
        k = ((p >> (3 * i)) & 7) % 7
        if 1 <= k <= 3:
            c, d, f = c + 2 * a, d + 2 * b, f + 2 * e + (k - 1)
        elif k >= 4:
            a, b, e = a + 2 * c, b + 2 * d, e + 2 * f + (k - 4)
    return a, b, c, d, e, f


def pack(co):
    a, b, c, d, e, f = co
    return a | b << 5 | c << 10 | d << 15 | e << 20 | f << 26


def unpack(t):
    return (t & 31, ((t << 22) & M) >> 27, ((t << 17) & M) >> 27, ((t << 12) & M) >> 27,
            ((t << 6) & M) >> 26, t >> 26)


TAB = [pack(compose4(p)) for p in range(4096)]


def test_coefficient_bounds_fit_the_packing():
    mx = [0] * 6
    for p in range(4096):
        for i, v in enumerate(compose4(p)):
            mx[i] = max(mx[i], v)
    assert mx == [29, 22, 22, 29, 40, 40]        # a, b, c, d, e, f
    assert all(unpack(pack(compose4(p))) == compose4(p) for p in range(4096))


def group_off4(w, g):
    bit = 12 * g
    wi, sh = bit >> 5, bit & 31
    if sh == 0:
        return (w[wi] << 2) & 0x3FFC
    if sh <= 20:
        return (w[wi] >> (sh - 2)) & 0x3FFC
    return (((w[wi + 1] << 32 | w[wi]) >> (sh - 2)) & M) & 0x3FFC


def walk64_table(w, x, y):
    for g in range(16):
        a, b, c, d, e, f = unpack(TAB[group_off4(w, g) >> 2])
        x, y = (b * y + a * x + e) & M, (d * y + c * x + f) & M
    return x, y


def test_table_walk_equals_definition_random():
    rng = np.random.default_rng(77)
    for _ in range(2000):
        w = [int(v) for v in rng.integers(0, 2 ** 32, 6, dtype=np.uint64)]
        x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
        assert walk64_table(w, x0, y0) == O.walk(1 << 32, x0, y0, np.array(w, np.uint32), 64)


def test_every_group_pattern_at_every_group_position():
    # each of the 4096 patterns in groups 0, 2 (straddles words 0/1), 5, 13, 15
    rng = np.random.default_rng(78)
    for g in (0, 2, 5, 13, 15):
        for p in range(0, 4096, 7):
            bits = int.from_bytes(rng.bytes(24), "little")
            bits &= ~(0xFFF << (12 * g))
            bits |= p << (12 * g)
            w = [(bits >> (32 * r)) & M for r in range(6)]
            x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
            assert walk64_table(w, x0, y0) == O.walk(1 << 32, x0, y0, np.array(w, np.uint32), 64)


def test_power_of_two_moduli_reduce_at_emission():
    # Z/2^32 -> Z/2^k is a ring homomorphism: the m = 2^k walk is the wrapped
    # walk reduced per coordinate (P15), so one table serves every m = 2^k
    rng = np.random.default_rng(79)
    for k in (8, 16, 20):
        for _ in range(200):
            w = [int(v) for v in rng.integers(0, 2 ** 32, 6, dtype=np.uint64)]
            x0, y0 = (int(v) for v in rng.integers(0, 2 ** k, 2, dtype=np.uint64))
            x, y = walk64_table(w, x0, y0)
            assert (x & ((1 << k) - 1), y & ((1 << k) - 1)) == O.walk(
                1 << k, x0, y0, np.array(w, np.uint32), 64)


# ---------------------------------------------------------------------------
# Bipartite variant: a group starts at an even global step,
# so it applies sigma, sigma^-1, sigma, sigma^-1; signed 5-5-5-5-6-6 fields.

def compose4_bip(p):
    a, b, e, c, d, f = 1, 0, 0, 0, 1, 0
    for i in range(4):
        k = ((p >> (3 * i)) & 7) % 7
        sg = -1 if i & 1 else 1
        if 1 <= k <= 3:
            c, d, f = c + sg * 2 * a, d + sg * 2 * b, f + sg * (2 * e + (k - 1))
        elif k >= 4:
            a, b, e = a + sg * 2 * c, b + sg * 2 * d, e + sg * (2 * f + (k - 4))
    return a, b, c, d, e, f


def pack_signed(co):
    a, b, c, d, e, f = co
    return (a & 31) | (b & 31) << 5 | (c & 31) << 10 | (d & 31) << 15 | (e & 63) << 20 | (f & 63) << 26


def sx(v, bits):
    return v - (1 << bits) if v >> (bits - 1) else v


def unpack_signed(t):
    return (sx(t & 31, 5), sx((t >> 5) & 31, 5), sx((t >> 10) & 31, 5), sx((t >> 15) & 31, 5),
            sx((t >> 20) & 63, 6), sx(t >> 26, 6))


TAB_BIP = [pack_signed(compose4_bip(p)) for p in range(4096)]


def test_bipartite_coefficient_bounds_fit_signed_fields():
    lo, hi = [0] * 6, [0] * 6
    for p in range(4096):
        for i, v in enumerate(compose4_bip(p)):
            lo[i], hi[i] = min(lo[i], v), max(hi[i], v)
    assert lo == [-7, -8, -8, -7, -12, -12] and hi == [5, 8, 8, 5, 14, 14]
    assert all(unpack_signed(TAB_BIP[p]) == compose4_bip(p) for p in range(4096))


def test_bipartite_table_walk_equals_definition():
    rng = np.random.default_rng(80)
    for _ in range(1000):
        w = [int(v) for v in rng.integers(0, 2 ** 32, 6, dtype=np.uint64)]
        x, y = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
        x0, y0 = x, y
        for g in range(16):
            a, b, c, d, e, f = unpack_signed(TAB_BIP[group_off4(w, g) >> 2])
            x, y = (b * y + a * x + e) & M, (d * y + c * x + f) & M
        rec = np.array(w, np.uint32)
        xs, ys = np.array([x0], np.uint64), np.array([y0], np.uint64)
        s0 = 64 * int(rng.integers(1, 1000))  # l0 + 64 j: even
        O.lib().or_walk_bipartite(1 << 32, xs.ctypes.data, ys.ctypes.data, rec.ctypes.data, 64, s0)
        assert (x, y) == (int(xs[0]), int(ys[0]))
