"""Multi-process (world size 2, gloo, CPU) tests of the sharding and all-reduce logic.

Each rank computes its shard with the CPU oracle (standing in for its GPU),
then the host-side decomposition (walker shards, global bulk indices, MC
thread shards, integer tally all-reduce) must reproduce the one-process
result exactly.  The GPU-side equivalence per shard is covered by
tests/test_gpu_mc.py::test_shards_sum_to_single_run.
"""
import os
import socket

import numpy as np
import torch.multiprocessing as mp

import oracle as O

M32 = 1 << 32


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_banerjeebk12_b200 import dist as gd
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # bulk: each rank generates its walkers' draws; gather by global index
        Wr, draws, seed = 16, 3, 42
        base, n = gd.walker_shard(rank, world, Wr)
        local = np.empty(Wr * draws, dtype=np.uint64)
        for t in range(n):
            local[t::Wr] = O.walker_draws(M32, 64, 64, seed, base + t, 0, draws)
        idx = gd.global_bulk_index(rank, world, Wr, np.arange(Wr * draws))
        full = torch.zeros(Wr * world * draws, dtype=torch.int64)
        full[torch.from_numpy(idx)] = torch.from_numpy(local.view(np.int64))
        dist.all_reduce(full)  # disjoint supports: the sum assembles the sequence
        # Monte Carlo: thread shards + exact integer all-reduce of tallies
        T = 32
        thread0, threads, total = gd.mc_shard(rank, world, T)
        r = O.mc_run(nthreads=threads, walker0=thread0, threads_total=total, photons_total=200,
                     D=48, seed=7)
        tal = gd.allreduce_tallies(r["tallies"].tolist())
        if rank == 0:
            q.put((full.numpy().view(np.uint64).copy(), tal))
    finally:
        dist.destroy_process_group()


def test_two_rank_shards_equal_single_process():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    bulk, tal = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # one process, W = 32 walkers
    assert np.array_equal(bulk, O.bulk(M32, 64, 64, 42, 32, 0, 32 * 3))
    whole = O.mc_run(nthreads=64, walker0=0, threads_total=64, photons_total=200, D=48, seed=7)
    assert tal == whole["tallies"].tolist()
    assert tal[0] == sum(tal[1:])
