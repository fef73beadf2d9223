"""Host FEED (csrc/feed.cpp) vs the oracle's seed-bit stream (R9), no GPU.

The feed is product code (vectorised SplitMix64 with non-temporal AVX-512
stores where the CPU has them, scalar multiversioned fallback); the oracle
computes the same counter-addressed words one by one.  Checked for
contiguous walker ranges, explicit walker lists (on-demand epochs over a
subset), odd word offsets and unaligned tails.
"""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SHIM = r'''
#include <cstdint>
namespace gg {
void feed_splitmix_rows(uint64_t, uint64_t, uint64_t, uint64_t, uint32_t, uint32_t *, uint64_t, bool,
                        double);
void feed_splitmix_rows_ids(uint64_t, uint64_t, const uint32_t *, uint64_t, uint64_t, uint32_t,
                            uint32_t *, uint64_t, bool, double);
}
extern "C" void run(uint64_t s, uint64_t t0, uint64_t n, uint64_t k0, uint32_t r, uint32_t *o,
                    uint64_t p, int nt, double pace) {
    gg::feed_splitmix_rows(s, t0, n, k0, r, o, p, nt != 0, pace);
}
extern "C" void run_ids(uint64_t s, uint64_t b, const uint32_t *ids, uint64_t n, uint64_t k0,
                        uint32_t r, uint32_t *o, uint64_t p, int nt, double pace) {
    gg::feed_splitmix_rows_ids(s, b, ids, n, k0, r, o, p, nt != 0, pace);
}
'''


@pytest.fixture(scope="module")
def feed(tmp_path_factory):
    d = tmp_path_factory.mktemp("feed")
    src, so = d / "shim.cpp", d / "shim.so"
    src.write_text(SHIM)
    feed_src = os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc", "feed.cpp")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-I",
                           os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc"),
                           "-I", "/usr/local/cuda/include", "-o", str(so), str(src), feed_src])
    return ctypes.CDLL(str(so))


def aligned(n_words):
    buf = np.zeros(n_words + 64, dtype=np.uint32)
    off = (-(buf.ctypes.data // 4)) % 8
    return buf, off


@pytest.mark.parametrize("pace", [0.0, 2e8])  # paced feed threads (bytes/s): same words
@pytest.mark.parametrize("nt", [0, 1])
@pytest.mark.parametrize("n,pitch,k0,rows", [(1000, 1024, 8, 6), (37, 64, 3, 6), (4096, 4096, 0, 12),
                                             (13, 32, 2, 1), (1 << 16, 1 << 16, 7, 4),
                                             (8192 + 37, 8192 + 64, 1, 3)])
def test_contiguous_rows(feed, n, pitch, k0, rows, nt, pace):
    buf, off = aligned(rows * pitch)
    seed, t0 = 0x5EED0002, 77
    ptr = buf.ctypes.data + off * 4
    feed.run(ctypes.c_uint64(seed), ctypes.c_uint64(t0), ctypes.c_uint64(n), ctypes.c_uint64(k0),
             ctypes.c_uint32(rows), ctypes.c_void_p(ptr), ctypes.c_uint64(pitch), ctypes.c_int(nt),
             ctypes.c_double(pace))
    got = buf[off:off + rows * pitch].reshape(rows, pitch)[:, :n]
    assert np.array_equal(got, O.stream_block(seed, t0, n, k0, rows))


def test_pacer_caps_the_store_rate(feed):
    """A paced feed thread writes no faster than its cap (prng_capi.cu
    feed_rate_for: the DMA of earlier chunks keeps its share of host memory)."""
    import time
    n, rows, pace = 1 << 16, 16, 4e8          # 4 MiB at 0.4 GB/s: >= 10.5 ms
    buf, off = aligned(rows * n)
    t = time.perf_counter()
    feed.run(ctypes.c_uint64(3), ctypes.c_uint64(0), ctypes.c_uint64(n), ctypes.c_uint64(0),
             ctypes.c_uint32(rows), ctypes.c_void_p(buf.ctypes.data + off * 4), ctypes.c_uint64(n),
             ctypes.c_int(1), ctypes.c_double(pace))
    assert time.perf_counter() - t >= rows * n * 4 / pace * 0.99


@pytest.mark.parametrize("nt", [0, 1])
@pytest.mark.parametrize("n,k0", [(1000, 8), (9, 5), (64, 0), (8192 + 9, 3)])
def test_walker_list_rows(feed, n, k0, nt):
    rows, pitch = 6, max(1024, (n + 63) // 64 * 64)
    buf, off = aligned(rows * pitch)
    ids = np.random.default_rng(n).permutation(20000)[:n].astype(np.uint32)
    feed.run_ids(ctypes.c_uint64(11), ctypes.c_uint64(500), ctypes.c_void_p(ids.ctypes.data),
                 ctypes.c_uint64(n), ctypes.c_uint64(k0), ctypes.c_uint32(rows),
                 ctypes.c_void_p(buf.ctypes.data + off * 4), ctypes.c_uint64(pitch), ctypes.c_int(nt),
                 ctypes.c_double(1e9 if nt else 0.0))
    got = buf[off:off + rows * pitch].reshape(rows, pitch)[:, :n]
    want = np.stack([O.stream_block(11, 500 + int(t), 1, k0, rows)[:, 0] for t in ids], axis=1)
    assert np.array_equal(got, want)


# ------------------------------------------------ f3: glibc rand_r seed bits
def test_oracle_rand_r_is_glibc():
    # the oracle's plain rand_r vs the system C library's (an independent
    # implementation of the paper's "LCG present in the glibc library")
    libc = ctypes.CDLL("libc.so.6")
    libc.rand_r.argtypes = [ctypes.POINTER(ctypes.c_uint)]
    for seed0 in (1, 12345, 0xFFFFFFFF, 0, 0x5EED0002):
        a = ctypes.c_uint(seed0)
        b = np.array([seed0], np.uint32)
        for _ in range(200):
            assert libc.rand_r(ctypes.byref(a)) == O.lib().or_rand_r(b.ctypes.data)
            assert a.value == int(b[0])


RANDR_SHIM = r'''
#include <cstdint>
namespace gg {
void feed_randr_rows(uint64_t, uint64_t, uint64_t, uint64_t, uint32_t, uint32_t *, uint64_t);
void feed_randr_rows_ids(uint64_t, uint64_t, const uint32_t *, uint64_t, uint64_t, uint32_t,
                         uint32_t *, uint64_t);
}
extern "C" void run(uint64_t s, uint64_t t0, uint64_t n, uint64_t k0, uint32_t r, uint32_t *o,
                    uint64_t p) { gg::feed_randr_rows(s, t0, n, k0, r, o, p); }
extern "C" void run_ids(uint64_t s, uint64_t b, const uint32_t *ids, uint64_t n, uint64_t k0,
                        uint32_t r, uint32_t *o, uint64_t p) {
    gg::feed_randr_rows_ids(s, b, ids, n, k0, r, o, p);
}
'''


@pytest.fixture(scope="module")
def randr_feed(tmp_path_factory):
    d = tmp_path_factory.mktemp("randr")
    src, so = d / "shim.cpp", d / "shim.so"
    src.write_text(RANDR_SHIM)
    feed_src = os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc", "feed.cpp")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-I",
                           os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc"),
                           "-I", "/usr/local/cuda/include", "-o", str(so), str(src), feed_src])
    return ctypes.CDLL(str(so))


@pytest.mark.parametrize("k0,rows", [(0, 8), (8, 6), (37, 3), (1000, 2)])
def test_randr_feed_jump_ahead_matches_plain_replay(randr_feed, k0, rows):
    n, pitch, seed, t0 = 50, 64, 0x5EED0001, 3
    buf = np.zeros(rows * pitch, np.uint32)
    randr_feed.run(ctypes.c_uint64(seed), ctypes.c_uint64(t0), ctypes.c_uint64(n), ctypes.c_uint64(k0),
                   ctypes.c_uint32(rows), ctypes.c_void_p(buf.ctypes.data), ctypes.c_uint64(pitch))
    got = buf.reshape(rows, pitch)[:, :n]
    for i in (0, 7, n - 1):
        for r in range(rows):
            assert got[r, i] == O.lib().or_stream_word32_randr(seed, t0 + i, k0 + r)
    ids = np.array([9, 2, 40], np.uint32)
    randr_feed.run_ids(ctypes.c_uint64(seed), ctypes.c_uint64(100), ctypes.c_void_p(ids.ctypes.data),
                       ctypes.c_uint64(3), ctypes.c_uint64(k0), ctypes.c_uint32(rows),
                       ctypes.c_void_p(buf.ctypes.data), ctypes.c_uint64(pitch))
    got = buf.reshape(rows, pitch)[:, :3]
    for i, t in enumerate(ids):
        for r in range(rows):
            assert got[r, i] == O.lib().or_stream_word32_randr(seed, 100 + int(t), k0 + r)


# ------------------------------------- f3: the generator itself as the FEED
GGCPU_SHIM = r'''
#include <cstdint>
#include "gg_internal.h"
extern "C" void run(uint64_t seed, uint64_t base, uint64_t l0, const uint32_t *ids, uint64_t n,
                    uint64_t k0, uint32_t r, uint32_t *o, uint64_t p, uint32_t *cx, uint32_t *cy,
                    uint32_t *cb, uint32_t *cn, uint64_t t0) {
    gg::GgCpuCache c{cx, cy, cb, cn, t0};
    gg::feed_ggcpu_rows(seed, base, l0, ids, n, k0, r, o, p, c);
}
'''


@pytest.fixture(scope="module")
def ggcpu_feed(tmp_path_factory):
    d = tmp_path_factory.mktemp("ggcpu")
    src, so = d / "shim.cpp", d / "shim.so"
    src.write_text(GGCPU_SHIM)
    feed_src = os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc", "feed.cpp")
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-I",
                           os.path.join(ROOT, "paper_conf_ipps_banerjeebk12_b200", "csrc"),
                           "-I", "/usr/local/cuda/include", "-o", str(so), str(src), feed_src])
    return ctypes.CDLL(str(so))


class _GgCache:
    def __init__(self, n):
        self.a = [np.zeros(n, np.uint32) for _ in range(4)]

    def args(self):
        return [ctypes.c_void_p(a.ctypes.data) for a in self.a]


def _ggcpu_rows(feed, cache, seed, base, l0, n, k0, rows, ids=None, t0=0):
    pitch = max(n, 1)
    buf = np.zeros(rows * pitch, np.uint32)
    feed.run(ctypes.c_uint64(seed), ctypes.c_uint64(base), ctypes.c_uint64(l0),
             ctypes.c_void_p(None if ids is None else ids.ctypes.data), ctypes.c_uint64(n),
             ctypes.c_uint64(k0), ctypes.c_uint32(rows), ctypes.c_void_p(buf.ctypes.data),
             ctypes.c_uint64(pitch), *cache.args(), ctypes.c_uint64(t0))
    return buf.reshape(rows, pitch)[:, :n]


def test_ggcpu_oracle_is_the_generator_reseeded_per_block():
    # R23 restated through the oracle's own Alg.1/Alg.2 (pinned elsewhere):
    # word k = x or y of label (k mod 64)/2 of walker t under seed_b
    seed, t = 0x5EED0001, 12
    for k in (0, 1, 7, 62, 63, 64, 65, 200):
        b, j = k // 64, (k % 64) // 2
        sb = O.lib().or_mix64(seed ^ (((b + 1) * 0xD1B54A32D192ED03) & (2**64 - 1)))
        lab = int(O.walker_draws(1 << 32, 64, 64, sb, t, 0, j + 1)[j])
        want = lab & 0xFFFFFFFF if k % 2 == 0 else lab >> 32
        assert O.lib().or_stream_word32_ggcpu(seed, t, k) == want


def test_ggcpu_feed_matches_oracle_sequential_random_and_lists(ggcpu_feed):
    seed, base, W = 0x5EED0007, 1000, 40
    cache = _GgCache(W)
    want = lambda t, k: O.lib().or_stream_word32_ggcpu(seed, base + t, k)  # noqa: E731
    # sequential row ranges (the bulk feed), crossing the 64-word block edges
    for k0, rows in ((0, 8), (8, 30), (38, 40), (78, 60)):
        got = _ggcpu_rows(ggcpu_feed, cache, seed, base, 0, W, k0, rows, t0=base)
        for t in (0, 5, W - 1):
            assert [int(v) for v in got[:, t]] == [want(t, k0 + r) for r in range(rows)]
    # backwards and odd starts (restart from the block's beginning)
    for k0, rows in ((3, 5), (129, 2), (64, 1), (65, 1)):
        got = _ggcpu_rows(ggcpu_feed, cache, seed, base, 0, W, k0, rows, t0=base)
        for t in (1, 17):
            assert [int(v) for v in got[:, t]] == [want(t, k0 + r) for r in range(rows)]
    # a sub-range of walkers (l0) and an explicit walker list
    got = _ggcpu_rows(ggcpu_feed, cache, seed, base, 20, 10, 140, 6, t0=base)
    assert [int(v) for v in got[:, 3]] == [want(23, 140 + r) for r in range(6)]
    ids = np.array([39, 0, 21, 7], np.uint32)
    got = _ggcpu_rows(ggcpu_feed, cache, seed, base, 0, 4, 146, 6, ids=ids, t0=base)
    for i, t in enumerate(ids):
        assert [int(v) for v in got[:, i]] == [want(int(t), 146 + r) for r in range(6)]
