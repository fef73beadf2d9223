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
