"""GPU list ranking (gg_list_rank) vs the oracle: ranks exact; FIS and splitter sets bit-exact.

Config C3 (BASELINE.json configs[2]): on-demand prng_next inside randomised
list ranking of a 2^24-node random linked list.  At 2^16 nodes the whole
randomised run is compared with the oracle's sequential replica
(or_lr_run); at 2^24 the ranks are compared with the definition (walking
the list) and the FIS invariants are checked on every round.
"""
import numpy as np
import pytest

import inputs
import oracle as O

pytestmark = pytest.mark.gpu
M32 = 1 << 32


def run_gpu(succ, pred, head, seed, want_sets=True):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    n = succ.size
    g = Generator(walkers=max(n, 1), seed=seed)
    s = torch.from_numpy(succ).cuda()
    p = torch.from_numpy(pred).cuda()
    rr = torch.empty(n, dtype=torch.int32, device="cuda") if want_sets else None
    sp = torch.empty(n, dtype=torch.int32, device="cuda") if want_sets else None
    rank, info = g.list_rank(s, p, head, removed_round=rr, is_splitter=sp)
    out = {"rank": rank.cpu().numpy(), "info": info}
    if want_sets:
        out["removed_round"] = rr.cpu().numpy()
        out["is_splitter"] = sp.cpu().numpy().astype(bool)
    g.close()
    return out


@pytest.mark.parametrize("n", [1, 2, 3, 5, 64, 1000, 4097, 1 << 16])
def test_full_parity_with_oracle_replica(n):
    succ, pred, head = inputs.random_list(n, 100 + n)
    seed = 0x5EED0003
    got = run_gpu(succ, pred, head, seed)
    want = O.lr_run(succ, pred, head, seed=seed)
    assert np.array_equal(got["rank"], O.lr_rank_seq(succ, head))
    assert np.array_equal(got["removed_round"], want["removed_round"])
    assert np.array_equal(got["is_splitter"], want["is_splitter"])
    info = got["info"]
    assert (info["rounds"], info["reduced"], info["splitters"], info["draws"]) == \
        (want["rounds"], want["reduced"], want["splitters"], want["draws"])


def test_ordered_list():
    succ, pred, head = inputs.ordered_list(50000)
    got = run_gpu(succ, pred, head, 1, want_sets=False)
    assert np.array_equal(got["rank"], np.arange(50000, dtype=np.int32))


def test_c3_full_size_ranks_and_fis_invariants():
    n = 1 << 24
    succ, pred, head = inputs.random_list(n, 0x5EED0003)
    got = run_gpu(succ, pred, head, 0x5EED0003)
    ref = O.lr_rank_seq(succ, head)
    assert np.array_equal(got["rank"], ref)
    rr = got["removed_round"]
    order = np.argsort(ref)  # list order
    info = got["info"]
    assert rr[order[0]] == -1 and rr[order[-1]] == -1
    assert (rr == -1).sum() == info["reduced"] <= -(-n // 24)
    for k in range(info["rounds"]):
        cur = order[(rr[order] == -1) | (rr[order] >= k)]
        gone = rr[cur] == k
        assert not np.any(gone[1:] & gone[:-1]), k          # independent set
        mu, sd = (cur.size - 2) / 8, np.sqrt((cur.size - 2) * 7 / 64)
        assert abs(gone.sum() - mu) < 6 * sd, k             # removal rate 1/8
    spl = got["is_splitter"]
    assert spl[order[0]] and np.all(rr[spl] == -1)
    # a sample of splitters is exact vs the oracle's draws: slot i of the
    # reduced list uses walker i, draw = rounds (R16', R18)
    reduced = np.flatnonzero(rr == -1)  # stable compaction keeps node-id order
    for i in list(range(0, reduced.size, reduced.size // 50)) + [reduced.size - 1]:
        lab = int(O.walker_draws(M32, 64, 64, 0x5EED0003, i, info["rounds"], 1)[0])
        v = reduced[i]
        assert bool(spl[v]) == (v == order[0] or (lab >> 58) == 0), i


class _FakeCollective:
    """Two ranks as two host threads of this process sharing one GPU: the
    gg_collective callbacks exchange through host copies behind a barrier.
    Exercises the sharded Phase II and the splitter exchange without NCCL."""

    def __init__(self, world):
        import threading
        self.world = world
        self.bar = threading.Barrier(world)
        self.slots = [None] * world

    def member(self, rank):
        import ctypes
        import torch
        from paper_conf_ipps_banerjeebk12_b200 import _lib
        from paper_conf_ipps_banerjeebk12_b200.dist import _device_view
        fc = self
        dev = torch.device("cuda", 0)

        def allgather(ctx, send, recv, nbytes):
            fc.slots[rank] = _device_view(send, nbytes, dev).cpu()
            fc.bar.wait()
            _device_view(recv, nbytes * fc.world, dev).copy_(torch.cat(fc.slots))
            torch.cuda.synchronize()
            fc.bar.wait()
            return 0

        def allreduce(ctx, buf, count):
            fc.slots[rank] = _device_view(buf, count * 4, dev).view(torch.int32).cpu()
            fc.bar.wait()
            tot = sum(s.to(torch.int64) for s in fc.slots).to(torch.int32)
            fc.bar.wait()
            _device_view(buf, count * 4, dev).view(torch.int32).copy_(tot)
            torch.cuda.synchronize()
            return 0

        class M:
            def __init__(self):
                self._ag = _lib.GG_ALLGATHER_FN(allgather)
                self._ar = _lib.GG_ALLREDUCE_I32_FN(allreduce)

            def struct(self):
                return _lib.gg_collective(rank, fc.world, self._ag, self._ar, None)
        return M()


@pytest.mark.parametrize("n,world", [(2, 2), (1000, 2), (1 << 16, 2), (1 << 16, 3), (200000, 4)])
def test_sharded_splitter_exchange(n, world):
    """world > 1: every rank ends with the exact ranks; FIS and splitter sets
    equal the one-GPU run (Phase I and the splitter choice are replicated)."""
    import threading
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    succ, pred, head = inputs.random_list(n, 7 + n)
    seed = 0x5EED0003
    single = run_gpu(succ, pred, head, seed)
    fc = _FakeCollective(world)
    res = [None] * world
    errs = []

    def worker(r):
        try:
            torch.cuda.set_device(0)
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                g = Generator(walkers=n, seed=seed)
                s = torch.from_numpy(succ).cuda()
                p = torch.from_numpy(pred).cuda()
                rr = torch.empty(n, dtype=torch.int32, device="cuda")
                sp = torch.empty(n, dtype=torch.int32, device="cuda")
                rank, info = g.list_rank(s, p, head, removed_round=rr, is_splitter=sp,
                                         stream=st, collective=fc.member(r))
                st.synchronize()
                res[r] = (rank.cpu().numpy(), rr.cpu().numpy(), sp.cpu().numpy().astype(bool), info)
                g.close()
        except Exception as e:  # pragma: no cover - surfaced below
            errs.append(e)
            fc.bar.abort()

    th = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not errs, errs
    ref = O.lr_rank_seq(succ, head)
    for r in range(world):
        rank, rr, sp, info = res[r]
        assert np.array_equal(rank, ref), r
        assert np.array_equal(rr, single["removed_round"]), r
        assert np.array_equal(sp, single["is_splitter"]), r
        assert info["splitters"] == single["info"]["splitters"]
