"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Configs (BASELINE.json): C1 = m 2^8, 1024 walkers, 2^20 numbers, in full;
C2 = m 2^32, 2^20 walkers, 2^30 uint32 numbers, in the launch configuration
bench.py times, checked on sampled walkers (every 1021st, all draws).
"""
import numpy as np
import pytest

import oracle as O
from conftest import read_golden

pytestmark = pytest.mark.gpu

M32 = 1 << 32


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    assert torch.cuda.is_available(), "GPU test needs CUDA"
    return torch


def G(**kw):
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    return Generator(**kw)


def as_u64(t):
    return t.cpu().numpy().view(np.uint64)


def test_worked_vectors_and_bulk_order(torch_cuda):
    torch = torch_cuda
    g = G(walkers=1024, seed=0, m=M32)
    out = torch.empty(3 * 1024, dtype=torch.int64, device="cuda")
    g.fill(out)
    z = as_u64(out)
    for row in read_golden("gg_full_generator.txt"):
        if row[0] == "bulk" or int(row[0]) != M32 or int(row[2]) < 0:
            continue
        t, j, val = int(row[1]), int(row[2]), int(row[3], 0)
        assert int(z[j * 1024 + t]) == val


def test_c1_full_parity_u64_then_u32(torch_cuda):
    torch = torch_cuda
    W, seed, m, n = 1024, 0x5EED0001, 256, 1 << 20
    want = O.bulk(m, 64, 64, seed, W, 0, n + 4096)
    g = G(walkers=W, seed=seed, m=m)
    out = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(out)
    assert np.array_equal(as_u64(out), want[:n])
    # U32 format: m^2 <= 2^32 -> one word per label, continuing the sequence
    o32 = torch.empty(4096, dtype=torch.int32, device="cuda")
    g.fill(o32)
    assert np.array_equal(o32.cpu().numpy().view(np.uint32).astype(np.uint64), want[n:])
    assert g.tell() == n + 4096


@pytest.mark.parametrize("epoch_draws", [1, 3, 16])
def test_chunked_ragged_fills_equal_one_fill(torch_cuda, epoch_draws):
    # fill(n1) + fill(n2) + ... == fill(n1 + n2 + ...) with n not multiples of W
    # (ragged tails) and streamed ring slots of 1, 3 and 16 draws.
    torch = torch_cuda
    W, seed = 1000, 77
    sizes = [1, 999, 1001, 2500, 7, 12345]
    total = sum(sizes)
    want = O.bulk(M32, 64, 64, seed, W, 0, total)
    g = G(walkers=W, seed=seed, m=M32, epoch_draws=epoch_draws)
    got = []
    for s in sizes:
        o = torch.empty(s, dtype=torch.int64, device="cuda")
        g.fill(o)
        got.append(as_u64(o))
    assert np.array_equal(np.concatenate(got), want)


def test_prefetched_window_equals_streamed(torch_cuda):
    torch = torch_cuda
    W, seed = 4096, 5
    n = W * 40 + 123
    a = G(walkers=W, seed=seed, epoch_draws=4)
    b = G(walkers=W, seed=seed, epoch_draws=4)
    b.prefetch(20)  # first 20 draws resident, the rest streamed
    oa = torch.empty(n, dtype=torch.int64, device="cuda")
    ob = torch.empty(n, dtype=torch.int64, device="cuda")
    a.fill(oa)
    b.fill(ob)
    assert torch.equal(oa, ob)
    t = 1234
    assert np.array_equal(as_u64(ob)[t::W][:40], O.walker_draws(M32, 64, 64, seed, t, 0, 40))


def test_u32_words_of_full_size_labels(torch_cuda):
    torch = torch_cuda
    W, seed = 512, 9
    g = G(walkers=W, seed=seed)
    o = torch.empty(2 * 3 * W, dtype=torch.int32, device="cuda")
    g.fill(o)
    lab = o.cpu().numpy().view(np.uint32).view(np.uint64)  # little-endian (x, y) pairs
    assert np.array_equal(lab, O.bulk(M32, 64, 64, seed, W, 0, 3 * W))


@pytest.mark.parametrize("m,l,l0", [(1000, 64, 64), (7, 64, 64), (1 << 16, 64, 64),
                                    ((1 << 30) - 35, 64, 64), (M32, 1, 64), (M32, 16, 8),
                                    (256, 11, 0), (M32, 100, 64), (2, 64, 64),
                                    # m above 2^30, not a power of two: 64-bit reduction
                                    ((1 << 32) - 5, 64, 64), ((1 << 31) + 11, 11, 7),
                                    ((3 << 30) + 1, 64, 64), ((1 << 30) + 3, 1, 64)])
def test_generic_m_and_l_parity(torch_cuda, m, l, l0):
    # General modulus (mod-m reduction each step) and walk lengths other
    # than 64 take the generic kernel; still bit-exact.
    torch = torch_cuda
    W, seed = 300, 31
    n = W * 5 + 17
    g = G(walkers=W, seed=seed, m=m, walk_len=l, burnin_len=l0)
    o = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert np.array_equal(as_u64(o), O.bulk(m, l, l0, seed, W, 0, n))


def test_c2_sampled_parity_bench_launch(torch_cuda):
    # C2 at full size, in the launch configuration bench.py times: prefetch
    # of all 512 draws, one prng_fill of 2^30 uint32 words.
    torch = torch_cuda
    W, seed = 1 << 20, 0x5EED0002
    g = G(walkers=W, seed=seed)
    g.prefetch(512)
    o = torch.empty(1 << 30, dtype=torch.int32, device="cuda")
    g.fill(o)
    torch.cuda.synchronize()
    lab = o.view(torch.int64).view(512, W)
    walkers = list(range(0, W, 1021)) + [W - 1]
    sub = lab[:, walkers].cpu().numpy().view(np.uint64)
    for i, t in enumerate(walkers[::8]):  # oracle budget: ~130 walkers x 512 draws
        assert np.array_equal(sub[:, i * 8], O.walker_draws(M32, 64, 64, seed, t, 0, 512)), t
    # property that holds at any size: every label's coordinates are 32-bit,
    # and no walker repeats its previous label in 512 draws (a stuck walk
    # would); the first draws of all walkers are distinct w.h.p.
    first = lab[0]
    assert torch.unique(first).numel() > W - 4


def test_callback_bits_match_oracle_walk(torch_cuda):
    # User-supplied bits (PRNG_BITS_CALLBACK): all-zero, all-ones and a
    # pattern; the oracle walks the same explicit words.
    torch = torch_cuda
    W, D = 64, 3

    def pattern(kind):
        def fn(walker0, nwalkers, word0, nwords):
            t = np.arange(walker0, walker0 + nwalkers, dtype=np.uint64)[None, :]
            k = np.arange(word0, word0 + nwords, dtype=np.uint64)[:, None]
            if kind == "zero":
                return np.zeros((nwords, nwalkers), np.uint32)
            if kind == "ones":
                return np.full((nwords, nwalkers), 0xFFFFFFFF, np.uint32)
            return ((t * np.uint64(2654435761) + k * np.uint64(40503) + np.uint64(12345))
                    & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        return fn

    for kind in ("zero", "ones", "pattern"):
        fn = pattern(kind)
        g = G(walkers=W, seed=0, bits_fn=fn)
        o = torch.empty(W * D, dtype=torch.int64, device="cuda")
        g.fill(o)
        z = as_u64(o)
        for t in (0, 5, W - 1):
            words = fn(t, 1, 0, 8 + 6 * D)[:, 0]
            x, y = O.walk(M32, int(words[0]), int(words[1]), words[2:8], 64)
            for j in range(D):
                x, y = O.walk(M32, x, y, words[8 + 6 * j: 14 + 6 * j], 64)
                assert int(z[j * W + t]) == O.label(M32, x, y), (kind, t, j)
        if kind == "zero":
            assert not z.any()  # (0,0) with b = 0 every step never moves
        if kind == "ones":
            assert np.all(z == np.uint64(0xFFFFFFFFFFFFFFFF))  # b = 7 -> stay (R4)


def test_mark_rewind_and_save_load(torch_cuda):
    torch = torch_cuda
    W = 2048
    g = G(walkers=W, seed=3)
    o = torch.empty(W * 5 + 11, dtype=torch.int64, device="cuda")
    g.fill(o)
    g.mark()
    blob = g.save()
    a = torch.empty(W * 7 + 5, dtype=torch.int64, device="cuda")
    g.fill(a)
    g.rewind()
    b = torch.empty_like(a)
    g.fill(b)
    assert torch.equal(a, b)
    h = G(walkers=W, seed=3)
    h.load(blob)
    c = torch.empty_like(a)
    h.fill(c)
    assert torch.equal(a, c)


def test_fill_host_matches_device_fill(torch_cuda):
    torch = torch_cuda
    W, seed, n = 4096, 11, 4096 * 37 + 3
    a = G(walkers=W, seed=seed, epoch_draws=8)
    b = G(walkers=W, seed=seed, epoch_draws=8)
    host = torch.empty(n, dtype=torch.int64).pin_memory()
    a.fill_host(host)
    d = torch.empty(n, dtype=torch.int64, device="cuda")
    b.fill(d)
    assert torch.equal(host, d.cpu())


def test_invalid_calls_have_no_side_effects(torch_cuda):
    torch = torch_cuda
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    g = G(walkers=256, seed=1)
    o = torch.empty(7, dtype=torch.int32, device="cuda")
    with pytest.raises(PrngError):
        g.fill(o)  # odd number of u32 words with m = 2^32
    assert g.tell() == 0
    g.epoch_begin(256, 2)
    with pytest.raises(PrngError):
        g.fill(torch.empty(4, dtype=torch.int64, device="cuda"))  # bulk inside an epoch
    g.epoch_end()


# ------------------------------------------------------------ f1 walk variants
@pytest.mark.parametrize("m,l", [(M32, 64), (256, 64), (1000, 64), (M32, 1), (1000, 1), (M32, 11),
                                 ((1 << 32) - 5, 64), ((3 << 30) + 1, 3)])
def test_bipartite_variant_parity(torch_cuda, m, l):
    torch = torch_cuda
    W, seed = 320, 13
    n = W * 6 + 7
    g = G(walkers=W, seed=seed, m=m, walk_len=l, variant=1)
    o = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert np.array_equal(as_u64(o), O.bulk_v(m, l, 64, 1, seed, W, 0, n))


@pytest.mark.parametrize("m", [M32, 1 << 16, 256])
def test_l1_fast_kernel_parity_ragged(torch_cuda, m):
    # l = 1 ("emit every vertex") takes the HBM-bound TMA kernel; ragged
    # fills, prefetched and streamed windows, u64 and u32 outputs.
    torch = torch_cuda
    W, seed = 1000, 5
    sizes = [1, 999, 40000, 12345, 31]
    total = sum(sizes)
    want = O.bulk(m, 1, 64, seed, W, 0, total)
    g = G(walkers=W, seed=seed, m=m, walk_len=1, epoch_draws=7)
    g.prefetch(20)
    got = []
    for s in sizes:
        o = torch.empty(s, dtype=torch.int64, device="cuda")
        g.fill(o)
        got.append(as_u64(o))
    assert np.array_equal(np.concatenate(got), want)
    if m <= 1 << 16:
        h = G(walkers=W, seed=seed, m=m, walk_len=1)
        o32 = torch.empty(total, dtype=torch.int32, device="cuda")
        h.fill(o32)
        assert np.array_equal(o32.cpu().numpy().view(np.uint32).astype(np.uint64), want)


def test_wide_modulus_on_demand_and_u32(torch_cuda):
    """m = 2^32 - 5 through prng_next (on demand) and the u32 word format."""
    torch = torch_cuda
    m, W, D, seed = (1 << 32) - 5, 200, 3, 91
    g = G(walkers=W, seed=seed, m=m)
    o32 = torch.empty(2 * W, dtype=torch.int32, device="cuda")
    g.fill(o32)  # draw 0 of every walker, 2 words per label (R12)
    g.epoch_begin(W, D)
    o = torch.empty(W * D, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=D, out=o)
    g.epoch_end()
    want = O.bulk(m, 64, 64, seed, W, 0, W * (D + 1)).reshape(D + 1, W)
    assert np.array_equal(o32.cpu().numpy().view(np.uint64), want[0])
    assert np.array_equal(o.view(W, D).cpu().numpy().view(np.uint64), want[1:].T)


def test_bipartite_on_demand(torch_cuda):
    torch = torch_cuda
    W, D, seed = 256, 4, 77
    g = G(walkers=W, seed=seed, variant=1)
    g.epoch_begin(W, D)
    o = torch.empty(W * D, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=D, out=o)
    g.epoch_end()
    z = o.view(W, D).cpu().numpy().view(np.uint64)
    want = O.bulk_v(M32, 64, 64, 1, seed, W, 0, W * D).reshape(D, W).T
    assert np.array_equal(z, want)


def test_randr_bit_source_parity(torch_cuda):
    # f3: paper-faithful glibc rand_r seed bits (bit_source 1), bulk + on-demand
    torch = torch_cuda
    W, seed = 256, 0x5EED0001
    g = G(walkers=W, seed=seed, bit_source=1, m=256)
    o = torch.empty(W * 4 + 3, dtype=torch.int64, device="cuda")
    g.fill(o)
    with O.bit_source(1):
        want = O.bulk(256, 64, 64, seed, W, 0, W * 4 + 3)
    assert np.array_equal(as_u64(o), want)


def test_ggcpu_bit_source_parity(torch_cuda):
    # f3: the generator itself, run by the host feed threads, supplies the
    # seed bits (bit_source 3, R23): streamed and prefetched bulk fills across
    # 64-word block edges, an on-demand epoch and an epoch over a walker list
    torch = torch_cuda
    W, seed = 300, 0x5EED0003
    g = G(walkers=W, seed=seed, bit_source=3, epoch_draws=5)
    n = W * 23 + 7  # draws 0..23: words 8..151, blocks 0..2
    o = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(o[: W * 11 + 5])
    g.fill(o[W * 11 + 5:])
    with O.bit_source(3):
        want = O.bulk(M32, 64, 64, seed, W, 0, n)
    assert np.array_equal(as_u64(o), want)
    g.close()
    g = G(walkers=W, seed=seed, bit_source=3)
    g.prefetch(12)
    o2 = torch.empty(W * 12, dtype=torch.int64, device="cuda")
    g.fill(o2)
    assert np.array_equal(as_u64(o2), want[: W * 12])
    # on demand: the next epoch starts at draw 12 (R10)
    g.epoch_begin(W, 3)
    od = torch.empty(W * 3, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=3, out=od)
    g.epoch_end()
    got = as_u64(od).reshape(W, 3) if od.numel() else None
    with O.bit_source(3):
        for t in (0, 1, 150, W - 1):
            assert np.array_equal(got[t], O.walker_draws(M32, 64, 64, seed, t, 12, 3)), t
    g.close()


@pytest.mark.parametrize("burnin", [64, 63])
def test_bipartite_fast_kernel_parity(torch_cuda, burnin):
    # variant 1 with l = 64 and m = 2^k takes the R2P (sigma, sigma^-1)-pair
    # kernel when every draw starts at an even global step (l0 even); an odd
    # l0 must fall back to the generic kernel.  Prefetched (K-mode) and
    # streamed fills, ragged walker count, u64 and u32 formats.
    torch = torch_cuda
    W, D, seed = 1000, 9, 0x5EED0009
    for m in (M32, 1 << 20):
        g = G(walkers=W, seed=seed, m=m, variant=1, burnin_len=burnin)
        g.prefetch(D)
        o = torch.empty(W * D - 3, dtype=torch.int64, device="cuda")
        g.fill(o)
        want = O.bulk_v(m, 64, burnin, 1, seed, W, 0, W * D + 5)
        assert np.array_equal(as_u64(o), want[: W * D - 3]), m
        o2 = torch.empty(8, dtype=torch.int64, device="cuda")  # streamed past the window
        g.fill(o2)
        assert np.array_equal(as_u64(o2), want[W * D - 3: W * D + 5]), m
        g.close()
    # on demand through prng_next
    g = G(walkers=W, seed=seed, variant=1, burnin_len=burnin)
    g.epoch_begin(W, 3)
    od = torch.empty(W * 3, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=3, out=od)
    g.epoch_end()
    got = as_u64(od).reshape(W, 3)
    want = O.bulk_v(M32, 64, burnin, 1, seed, W, 0, W * 3).reshape(3, W).T
    assert np.array_equal(got, want)
    g.close()


def test_any_walk_length_parity(torch_cuda):
    # gg_fill_any_kernel / gg_walk_r2p_any: every last-group size (l mod 10 =
    # 0..9, single-step tails), records ending inside / exactly at a word, for
    # bulk fills and prng_next
    torch = torch_cuda
    W, D, seed = 97, 3, 0x5EED000A
    for l in list(range(2, 42)) + [63, 65, 100, 128, 333]:
        g = G(walkers=W, seed=seed, walk_len=l, m=1 << 16)
        o = torch.empty(W * D, dtype=torch.int64, device="cuda")
        g.fill(o)
        want = O.bulk_v(1 << 16, l, 64, 0, seed, W, 0, W * (D + 2))
        assert np.array_equal(as_u64(o), want[: W * D]), l
        g.epoch_begin(W, 2)
        od = torch.empty(W * 2, dtype=torch.int64, device="cuda")
        g.consume(W, uniform=2, out=od)
        g.epoch_end()
        assert np.array_equal(as_u64(od).reshape(W, 2), want[W * D:].reshape(2, W).T), l
        g.close()


@pytest.mark.parametrize("m", [3, 1000, 65521, (1 << 30) - 35, 1 << 30])
def test_non_power_of_two_fast_kernel_parity(torch_cuda, m):
    # m <= 2^30 not a power of two takes the R2P kernel with two conditional
    # subtracts per step (bulk, u64 and u32 formats, and prng_next)
    torch = torch_cuda
    W, D, seed = 700, 5, 0x5EED000B
    g = G(walkers=W, seed=seed, m=m)
    g.prefetch(D)
    o = torch.empty(W * D - 1, dtype=torch.int64, device="cuda")
    g.fill(o)
    want = O.bulk_v(m, 64, 64, 0, seed, W, 0, W * D + 2 * W)
    assert np.array_equal(as_u64(o), want[: W * D - 1])
    if m <= 65536:
        g2 = G(walkers=W, seed=seed, m=m)
        o32 = torch.empty(W * D, dtype=torch.int32, device="cuda")
        g2.fill(o32)
        assert np.array_equal(o32.cpu().numpy().view(np.uint32).astype(np.uint64), want[: W * D])
        g2.close()
    g.close()
    g = G(walkers=W, seed=seed, m=m)  # on demand from draw 0 (a ragged fill would skip draws, R10)
    g.epoch_begin(W, 2)
    od = torch.empty(W * 2, dtype=torch.int64, device="cuda")
    g.consume(W, uniform=2, out=od)
    g.epoch_end()
    assert np.array_equal(as_u64(od).reshape(W, 2), want[: 2 * W].reshape(2, W).T)
    g.close()


# ------------------------------------------- 32-bit draw cursor, checkpoints
def test_draw_index_limit_refused_without_side_effects(torch_cuda):
    """Draw indices are 32-bit in the kernels: a fill or prefetch whose end
    passes 2^32 - 256 draws (the kernels' loop margin) is refused with
    PRNG_E_UNSUPPORTED before anything is enqueued.  Up
    to the limit the numbers are still the oracle's: a walk of draw J's
    record (stream words 2 + R0 + 6J .., R9) from the saved walker state
    (checkpoint resume at N = J*W)."""
    import struct
    torch = torch_cuda
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    W, seed = 64, 5
    g = G(walkers=W, seed=seed)
    blob = bytearray(g.save())
    J = (1 << 32) - 256 - 3
    struct.pack_into("<Q", blob, 16, J * W)          # SavedHeader.N
    g.load(bytes(blob))
    assert g.tell() == J * W
    big = torch.full((4 * W,), 7, dtype=torch.int64, device="cuda")
    for call in (lambda: g.fill(big), lambda: g.prefetch(4),
                 lambda: g.fill_host(torch.empty(4 * W, dtype=torch.int64).pin_memory())):
        with pytest.raises(PrngError) as e:
            call()
        assert e.value.status == -2  # PRNG_E_UNSUPPORTED
    torch.cuda.synchronize()
    assert g.tell() == J * W and bool((big == 7).all())
    # draws J .. J+2 (end = 2^32 - 256, the limit): OK, oracle-exact
    g.fill(big, n=3 * W)
    assert g.tell() == (J + 3) * W
    z = as_u64(big[:3 * W]).reshape(3, W)
    hdr = 12 * 8
    xs = np.frombuffer(bytes(blob), dtype=np.uint32, count=W, offset=hdr)
    ys = np.frombuffer(bytes(blob), dtype=np.uint32, count=W, offset=hdr + 4 * W)
    for t in (0, 37, W - 1):
        x, y = int(xs[t]), int(ys[t])
        for d in range(3):
            k0 = 2 + 6 + 6 * (J + d)
            rec = [O.stream_word32(seed, t, k0 + r) for r in range(6)]
            x, y = O.walk(M32, x, y, rec, 64)
            assert int(z[d, t]) == O.label(M32, x, y), (t, d)
    with pytest.raises(PrngError) as e:
        g.fill(big, n=1)                               # one draw past the limit
    assert e.value.status == -2
    assert g.tell() == (J + 3) * W
    g.close()


@pytest.mark.parametrize("other", [dict(walker_base=64), dict(variant=1), dict(burnin_len=32),
                                   dict(bit_source=1)])
def test_checkpoint_refused_by_a_different_stream(torch_cuda, other):
    """prng_load only into a handle that selects the same bit streams and walk
    (rank 1 must not load rank 0's checkpoint silently)."""
    from paper_conf_ipps_banerjeebk12_b200 import PrngError
    W, seed = 64, 9
    a = G(walkers=W, seed=seed)
    blob = a.save()
    b = G(walkers=W, seed=seed, **other)
    with pytest.raises(PrngError) as e:
        b.load(blob)
    assert e.value.status == -1
    assert b.tell() == 0
    c = G(walkers=W, seed=seed)
    c.load(blob)  # the same configuration loads
    a.close(), b.close(), c.close()
