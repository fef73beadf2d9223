"""GPU parity for C5 (BASELINE.json: "2^34 numbers sharded over 1/2/4/8 B200
with disjoint seed-bit streams").

Sharding rule: GPU r of G owns the global walkers
[r·W/G, (r+1)·W/G); every label is a pure function of (seed, global walker,
draw) (R9, R11), so the union of the shards' outputs is the single-GPU output
re-interleaved by walker.  Checked (i) exactly on a small sweep over G = 1, 2,
4, 8 through both the streamed (E-mode) and the prefetched (K-mode) fill, and
(ii) against the oracle on sampled walkers of one full-size C5 fill in the
launch configuration `bench.py --workload c5` times (rank 3 of 8: 2^20
walkers from global id 3·2^20, a 2 GiB buffer of 2^28 labels = 256 draws).
"""
import numpy as np
import pytest

import oracle as O

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


@pytest.mark.parametrize("prefetch", [False, True])
def test_shard_union_equals_single_gpu(torch_cuda, prefetch):
    torch = torch_cuda
    W, D, seed = 4096 + 64, 40, 0x5EED0005  # W divisible by 8, not by 32 per shard
    single = G(walkers=W, seed=seed)
    ref = torch.empty(W * D, dtype=torch.int64, device="cuda")
    single.fill(ref)
    ref = ref.view(D, W).cpu()
    for world in (1, 2, 4, 8):
        Wr = W // world
        for r in range(world):
            g = G(walkers=Wr, seed=seed, walker_base=r * Wr, epoch_draws=8)
            out = torch.empty(Wr * D, dtype=torch.int64, device="cuda")
            if prefetch:
                g.prefetch(D)
            # two ragged chunks: the shard's sequence does not depend on chunking
            n0 = Wr * 7 + 13
            g.fill(out[:n0])
            g.fill(out[n0:])
            assert torch.equal(out.view(D, Wr).cpu(), ref[:, r * Wr:(r + 1) * Wr]), (world, r)
            g.close()


def test_c5_full_size_fill_sampled_parity(torch_cuda):
    torch = torch_cuda
    world, rank, seed = 8, 3, 0x5EED0005
    Wr = (1 << 23) // world
    base = rank * Wr
    D = (1 << 28) // Wr  # 256 draws per walker per fill
    g = G(walkers=Wr, seed=seed, walker_base=base)
    out = torch.empty(1 << 28, dtype=torch.int64, device="cuda")
    # second fill of the job (draws 256..511), as bench.py's chunk loop runs it
    g.prefetch(D)
    g.fill(out)
    g.prefetch(D)
    g.fill(out)
    torch.cuda.synchronize()
    lab = out.view(D, Wr)
    local = list(range(0, Wr, 8191)) + [Wr - 1]
    sub = lab[:, local].cpu().numpy().view(np.uint64)
    for i, t in enumerate(local):  # ~130 walkers x 256 draws of oracle work
        want = O.walker_draws(M32, 64, 64, seed, base + t, D, D)
        assert np.array_equal(sub[:, i], want), t
    assert torch.unique(lab[0]).numel() > Wr - 4
    g.close()
