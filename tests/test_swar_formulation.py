"""Host-side check of the kernel's SWAR step formulation (no GPU).

gg_walk64 (include/prng_device.cuh) does not evaluate the Gabber-Galil step
the way the paper writes it; it repacks the 192-bit record into 10-field
words, derives move masks and constants with word-parallel logic and uses
u = x + y + c so that either move is one add.  This test re-expresses that
exact instruction-level recipe in Python (32-bit wrap-around, the same
shifts, masks and multiply-high) and checks it against the oracle's plain
step-by-step walk on random records — including the masking bug class where
garbage bits of MY leak into C.  The GPU parity tests then check that the
CUDA code implements this recipe.
"""
import numpy as np

import oracle as O

M = 0xFFFFFFFF


def _word10(Q, nk, x, y):
    f1, f2 = Q >> 1, Q >> 2
    MY = ((f1 | Q) & 0x09249249) & ~f2 & M
    MX = (f2 & ~(f1 & Q)) & M
    C = (Q - MY) & M
    for k in range(nk):
        py, px = MY & (1 << 3 * k), MX & (1 << 3 * k)
        ct = (C << (30 - 3 * k)) & M          # IMAD.SHL
        c = ct >> 30                         # LEA.HI operand
        u = (x + y + c) & M
        if py:
            y = (u + x) & M
        if px:
            x = (u + y) & M
    return x, y


def _fsr(lo, hi, s):
    return ((hi << 32 | lo) >> s) & M


def walk64_swar(w, x, y):
    x, y = _word10(w[0], 10, x, y)
    for a, s in [(0, 30), (1, 28), (2, 26), (3, 24), (4, 22)]:
        x, y = _word10(_fsr(w[a], w[a + 1], s), 10, x, y)
    return _word10(w[5] >> 20, 4, x, y)


def test_swar_recipe_equals_definition_random():
    rng = np.random.default_rng(2024)
    for _ in range(2000):
        w = [int(v) for v in rng.integers(0, 2 ** 32, 6, dtype=np.uint64)]
        x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
        assert walk64_swar(w, x0, y0) == O.walk(1 << 32, x0, y0, np.array(w, np.uint32), 64)


def test_swar_recipe_every_field_value_at_every_position():
    # each 3-bit value 0..7 at each of the 64 field positions, others random
    rng = np.random.default_rng(5)
    for i in range(64):
        for b in range(8):
            bits = int.from_bytes(rng.bytes(24), "little")
            bits &= ~(7 << (3 * i))
            bits |= b << (3 * i)
            w = [(bits >> (32 * r)) & M for r in range(6)]
            x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
            assert walk64_swar(w, x0, y0) == O.walk(1 << 32, x0, y0, np.array(w, np.uint32), 64)


# ---------------------------------------------------------------------------
# R2P form (gg_word10_r2p / gg_word10x2_r2p): the step predicates are not
# tested bit by bit; R2P PR, S.Bn, mask loads predicate register P_i from bit
# i (i = 0..6) of byte n of S.  Model exactly that: for each group the kernel
# names a source (F or G = F >> 6), a byte and the bit offsets of py/px inside
# the byte; the step then reads P[bit] of that byte only.  A wrong byte, a
# flag outside bits 0..6 of its byte, or a wrong G shift fails here.

def _r2p_load(S, byte):
    v = (S >> (8 * byte)) & 0xFF
    return [(v >> i) & 1 for i in range(7)]  # P0..P6 (bit 7 is not loadable)


# (source, step k, bit of py within S) for the 10-field word, as in
# gg_word10_r2p with G = F >> 4: F.B0 0,1 | G.B0 2,3 | G.B1 4,5 | F.B2 6,7 | F.B3 8,9
G_SHIFT = 4
R2P_GROUPS_10 = [("F", 0, 0), ("F", 1, 3), ("G", 2, 2), ("G", 3, 5), ("G", 4, 8),
                 ("G", 5, 11), ("F", 6, 18), ("F", 7, 21), ("F", 8, 24), ("F", 9, 27)]
R2P_GROUPS_4 = [("F", 0, 0), ("F", 1, 3), ("G", 2, 2), ("G", 3, 5)]


def _word10_r2p(Q, nk, x, y):
    f1, f2 = Q >> 1, Q >> 2
    MY = ((f1 | Q) & 0x09249249) & ~f2 & M
    MX = (f2 & ~(f1 & Q)) & M
    C = (Q - MY) & M
    F = (MY | ((MX << 1) & 0x12492492)) & M
    G = F >> G_SHIFT
    for src, k, bit in (R2P_GROUPS_10 if nk == 10 else R2P_GROUPS_4):
        S = F if src == "F" else G
        byte, off = bit // 8, bit % 8
        assert off + 1 <= 6, "flag outside the 7 loadable bits of the byte"
        P = _r2p_load(S, byte)
        py, px = P[off], P[off + 1]
        c = ((C << (30 - 3 * k)) & M) >> 30
        u = (x + y + c) & M
        if py:
            y = (u + x) & M
        if px:
            x = (u + y) & M
    return x, y


def walk64_r2p(w, x, y):
    x, y = _word10_r2p(w[0], 10, x, y)
    for a, s in [(0, 30), (1, 28), (2, 26), (3, 24), (4, 22)]:
        x, y = _word10_r2p(_fsr(w[a], w[a + 1], s), 10, x, y)
    return _word10_r2p(w[5] >> 20, 4, x, y)


def test_r2p_groups_cover_each_step_once_in_order():
    for groups, nk in ((R2P_GROUPS_10, 10), (R2P_GROUPS_4, 4)):
        assert [k for _, k, _ in groups] == list(range(nk))
        for src, k, bit in groups:  # the flags of step k sit at 3k (F) or 3k - G_SHIFT (G)
            assert bit == (3 * k if src == "F" else 3 * k - G_SHIFT)
        # steps are paired: each R2P (source, byte) loads the flags of two steps
        loads = {}
        for src, k, bit in groups:
            loads.setdefault((src, bit // 8), []).append(k)
        assert all(len(v) == 2 for v in loads.values()), loads
        assert len(loads) == nk // 2


def test_r2p_recipe_every_field_value_at_every_position():
    rng = np.random.default_rng(11)
    for i in range(64):
        for b in range(8):
            bits = int.from_bytes(rng.bytes(24), "little")
            bits &= ~(7 << (3 * i))
            bits |= b << (3 * i)
            w = [(bits >> (32 * r)) & M for r in range(6)]
            x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
            assert walk64_r2p(w, x0, y0) == O.walk(1 << 32, x0, y0, np.array(w, np.uint32), 64)


# ---------------------------------------------------------------------------
# Bipartite variant (gg_r2p_two_bip): in every R2P pair the
# first step (even field index = even global step) applies sigma_k and the
# second sigma_k^{-1}: r = 2x + c, @py y -= r | v = 2y + c, @px x -= v.

def _word10_r2p_bip(Q, nk, x, y):
    f1, f2 = Q >> 1, Q >> 2
    MY = ((f1 | Q) & 0x09249249) & ~f2 & M
    MX = (f2 & ~(f1 & Q)) & M
    C = (Q - MY) & M
    F = (MY | ((MX << 1) & 0x12492492)) & M
    G = F >> G_SHIFT
    for src, k, bit in (R2P_GROUPS_10 if nk == 10 else R2P_GROUPS_4):
        S = F if src == "F" else G
        P = _r2p_load(S, bit // 8)
        py, px = P[bit % 8], P[bit % 8 + 1]
        c = ((C << (30 - 3 * k)) & M) >> 30
        if k % 2 == 0:
            u = (x + y + c) & M
            if py:
                y = (u + x) & M
            if px:
                x = (u + y) & M
        else:
            r, v = (2 * x + c) & M, (2 * y + c) & M
            if py:
                y = (y - r) & M
            if px:
                x = (x - v) & M
    return x, y


def walk64_r2p_bip(w, x, y):
    x, y = _word10_r2p_bip(w[0], 10, x, y)
    for a, s in [(0, 30), (1, 28), (2, 26), (3, 24), (4, 22)]:
        x, y = _word10_r2p_bip(_fsr(w[a], w[a + 1], s), 10, x, y)
    return _word10_r2p_bip(w[5] >> 20, 4, x, y)


def _oracle_bip(w, x0, y0, s0):
    rec = np.array(w, np.uint32)
    xs, ys = np.array([x0], np.uint64), np.array([y0], np.uint64)
    O.lib().or_walk_bipartite(1 << 32, xs.ctypes.data, ys.ctypes.data, rec.ctypes.data, 64, s0)
    return int(xs[0]), int(ys[0])


def test_r2p_bipartite_recipe_every_field_value_at_every_position():
    rng = np.random.default_rng(13)
    for i in range(64):
        for b in range(8):
            bits = int.from_bytes(rng.bytes(24), "little")
            bits &= ~(7 << (3 * i))
            bits |= b << (3 * i)
            w = [(bits >> (32 * r)) & M for r in range(6)]
            x0, y0 = (int(v) for v in rng.integers(0, 2 ** 32, 2, dtype=np.uint64))
            s0 = 64 * int(rng.integers(1, 1000))  # l0 + 64 j: even
            assert walk64_r2p_bip(w, x0, y0) == _oracle_bip(w, x0, y0, s0)
