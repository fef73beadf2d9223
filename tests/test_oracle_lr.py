"""Pins for the list-ranking oracle (§V; no GPU).

The final ranks are randomness-independent and must equal the definition
("distance of any node ... from either end of the list", R17: from the head)
computed by walking the list.  The randomised phases are pinned by the
invariants the paper states or implies: every Phase I round removes an
independent set (FIS), head and tail are never removed (R14), an
interior node leaves w.p. 1/8 per round (b(u)=1, both neighbours 0), and
the loop stops at n / log n nodes (Alg.3 output).
"""
import numpy as np
import pytest

import inputs
import oracle as O


@pytest.mark.parametrize("n", [1, 2, 3, 4, 17, 1000, 1 << 14])
@pytest.mark.parametrize("kind", ["random", "ordered"])
def test_ranks_equal_sequential_definition(n, kind):
    succ, pred, head = inputs.random_list(n, 11) if kind == "random" else inputs.ordered_list(n)
    ref = O.lr_rank_seq(succ, head)
    # the definition itself: head 0, each successor one more
    assert ref[head] == 0
    nz = succ >= 0
    assert np.all(ref[succ[nz]] == ref[nz] + 1)
    r = O.lr_run(succ, pred, head, seed=7)
    assert np.array_equal(r["rank"], ref)


def _order(succ, head):
    out, v = [], head
    while v >= 0:
        out.append(v)
        v = succ[v]
    return np.array(out)


def test_fis_invariants_and_removal_rate():
    n = 1 << 16
    succ, pred, head = inputs.random_list(n, 3)
    r = O.lr_run(succ, pred, head, seed=1234)
    rr = r["removed_round"]
    order = _order(succ, head)
    tail = order[-1]
    assert rr[head] == -1 and rr[tail] == -1
    L = int(np.floor(np.log2(n)))
    target = -(-n // L)
    assert r["reduced"] <= target
    assert (rr == -1).sum() == r["reduced"]
    alive_before = n
    for k in range(r["rounds"]):
        # list at the start of round k = nodes not removed before k, in list order
        cur = order[(rr[order] == -1) | (rr[order] >= k)]
        assert cur.size == alive_before
        gone = rr[cur] == k
        # independent set: no two list-adjacent nodes leave in the same round
        assert not np.any(gone[1:] & gone[:-1])
        # Pr[remove] = 1/8 for interior nodes (3 independent fair bits)
        interior = cur.size - 2
        mu, sd = interior / 8, np.sqrt(interior * (1 / 8) * (7 / 8))
        assert abs(gone.sum() - mu) < 5 * sd + 1, (k, gone.sum(), mu)
        alive_before -= int(gone.sum())
    # the previous round still had more than the target
    assert r["rounds"] == 0 or r["reduced"] + (rr == r["rounds"] - 1).sum() > target
    # splitters: head + ~1/64 of the reduced list
    spl = r["is_splitter"]
    assert spl[head] and spl.sum() == r["splitters"]
    assert np.all(rr[spl] == -1)
    A = r["reduced"]
    assert abs((spl.sum() - 1) - A / 64) < 5 * np.sqrt(A / 64) + 1
    # draws: one per active node per round + one per reduced node (~7.7n at large n)
    assert r["draws"] == sum(int(((rr == -1) | (rr >= k)).sum()) for k in range(r["rounds"])) + A


def test_bits_really_drive_the_fis():
    # Different generator seeds give different FIS sets but identical ranks.
    n = 4096
    succ, pred, head = inputs.random_list(n, 9)
    a = O.lr_run(succ, pred, head, seed=1)
    b = O.lr_run(succ, pred, head, seed=2)
    assert not np.array_equal(a["removed_round"], b["removed_round"])
    assert np.array_equal(a["rank"], b["rank"])
