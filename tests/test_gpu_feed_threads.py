"""Determinism contract: the numbers do not depend on the
number of host FEED threads.  The feed threads claim 4096-walker blocks of
each pinned chunk from a shared counter (prng_capi.cu feed_chunk), so which
thread writes which block changes from run to run; the bits of a block are a
pure function of (seed, walker, word) (R9).  Ragged walker counts spanning
several blocks, bulk fills streamed by the feed, an on-demand epoch over a
walker list and a small list ranking, for 1 / 3 / 7 / 16 threads, against the
oracle."""
import numpy as np
import pytest

import inputs
import oracle as O

pytestmark = pytest.mark.gpu
M32 = 1 << 32
W = 3 * 4096 + 123
SEED = 0x5EED00F7


@pytest.fixture(scope="module")
def want_bulk():
    n = 2 * W + 5
    return O.bulk(M32, 64, 64, SEED, W, 0, n)


@pytest.mark.parametrize("threads", [1, 3, 7, 16])
def test_bulk_and_on_demand_independent_of_feed_threads(threads, want_bulk):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    g = Generator(walkers=W, seed=SEED, host_threads=threads, epoch_draws=2)
    o = torch.empty(want_bulk.size, dtype=torch.int64, device="cuda")
    g.fill(o)
    assert np.array_equal(o.cpu().numpy().view(np.uint64), want_bulk)
    # on-demand epoch over every 5th walker, one draw each (walker-list feed)
    ids = np.arange(0, W, 5, dtype=np.uint32)
    g.epoch_begin_list(ids, 1)
    od = torch.empty(ids.size, dtype=torch.int64, device="cuda")
    g.consume(ids.size, uniform=1, out=od)
    g.epoch_end()
    got = od.cpu().numpy().view(np.uint64)
    J0 = -(-want_bulk.size // W)  # R10: the epoch starts at the next whole draw
    lib = O.lib()
    for k in (0, 1, ids.size // 2, ids.size - 1):
        t = int(ids[k])
        x, y = O.walker_init(M32, 64, SEED, t)
        xa, ya = np.array([x], np.uint64), np.array([y], np.uint64)
        # the walker's bulk draws, then draw J0 (R10: the rest of draw J0-1 is skipped)
        for j in range((want_bulk.size - t + W - 1) // W):
            lib.or_walker_draw(M32, 64, 64, SEED, t, j, xa.ctypes.data, ya.ctypes.data)
        want = int(lib.or_walker_draw(M32, 64, 64, SEED, t, J0, xa.ctypes.data, ya.ctypes.data))
        assert int(got[k]) == want, (threads, k)
    g.close()


@pytest.mark.parametrize("threads", [1, 5, 16])
def test_list_ranking_independent_of_feed_threads(threads):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    n = 40000  # rounds with prefed windows over several feed blocks
    succ, pred, head = inputs.random_list(n, 77)
    g = Generator(walkers=n, seed=0x5EED0003, host_threads=threads)
    rr = torch.empty(n, dtype=torch.int32, device="cuda")
    rank, info = g.list_rank(torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda(), head,
                             removed_round=rr)
    g.close()
    want = O.lr_run(succ, pred, head, seed=0x5EED0003)
    assert np.array_equal(rank.cpu().numpy(), O.lr_rank_seq(succ, head))
    assert np.array_equal(rr.cpu().numpy(), want["removed_round"])
    assert info["draws"] == want["draws"]
