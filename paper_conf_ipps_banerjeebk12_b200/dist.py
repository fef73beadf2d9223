"""Multi-GPU plumbing: walker shards and the one collective the path needs.

One process per GPU (torch.distributed, NCCL over NVLink on the GPU box,
gloo in the CPU tests).  The generator shards naturally: GPU r owns global
walkers [r*W, (r+1)*W) and therefore disjoint seed-bit streams (reading R9:
a walker's stream depends only on its global id), so bulk generation needs
no communication and the union over GPUs equals the one-GPU output walker by
walker (§I-B: "Each thread performing the walk is essentially executing
independent of other threads").  The Monte Carlo consumer (§VI) sums
integer fixed-point tallies across GPUs with one all-reduce; sums of int64
are exact and order independent, so the sharded result equals the one-GPU
result bit for bit.
"""
from __future__ import annotations


def walker_shard(rank: int, world: int, walkers_per_rank: int):
    """(walker_base, walkers) of rank `rank` for weak scaling (fixed walkers per GPU)."""
    if not 0 <= rank < world:
        raise ValueError("rank out of range")
    return rank * walkers_per_rank, walkers_per_rank


def global_bulk_index(rank: int, world: int, walkers_per_rank: int, local_index):
    """Map a shard's local bulk position g = j*W + t to the position of the same
    (walker, draw) in the one-GPU sequence over W*world walkers (reading R11)."""
    W = walkers_per_rank
    j = local_index // W
    t = local_index % W
    return j * (W * world) + rank * W + t


def mc_shard(rank: int, world: int, threads_per_rank: int):
    """(thread0, threads, threads_total) for gg_mc_run on rank `rank`."""
    base, n = walker_shard(rank, world, threads_per_rank)
    return base, n, threads_per_rank * world


def allreduce_tallies(tallies, group=None, device=None):
    """Exact integer sum of Monte Carlo tallies over all ranks (SUM all-reduce)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor(list(tallies), dtype=torch.int64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return [int(v) for v in t.cpu().tolist()]


def _device_view(ptr: int, nbytes: int, device):
    """A uint8 CUDA tensor aliasing `nbytes` at device address `ptr`."""
    import torch

    class _Buf:
        __cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                    "version": 3, "strides": None}
    return torch.as_tensor(_Buf(), device=device)


class Collective:
    """gg_collective backed by torch.distributed (NCCL over NVLink on the GPU
    box; gloo in tests).  Keep the object alive for the duration of the call."""

    def __init__(self, group=None, device=None):
        import torch
        import torch.distributed as dist
        from . import _lib
        self.group = group
        self.device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        # NCCL works on the device buffers in place; other backends (gloo in
        # the single-GPU multi-rank tests) go through host copies.
        on_dev = dist.get_backend(group) == "nccl"
        self.errors = []

        def allgather(ctx, send, recv, nbytes):
            try:
                s = _device_view(send, nbytes, self.device)
                r = _device_view(recv, nbytes * self.world, self.device)
                if on_dev:
                    dist.all_gather_into_tensor(r, s, group=self.group)
                else:
                    rh = torch.empty(nbytes * self.world, dtype=torch.uint8)
                    dist.all_gather_into_tensor(rh, s.cpu(), group=self.group)
                    r.copy_(rh)
                torch.cuda.synchronize(self.device)
                return 0
            except Exception as e:  # errors cannot cross the C ABI as exceptions
                self.errors.append(e)
                return -1

        def allreduce_i32(ctx, buf, count):
            try:
                b = _device_view(buf, count * 4, self.device).view(torch.int32)
                if on_dev:
                    dist.all_reduce(b, op=dist.ReduceOp.SUM, group=self.group)
                else:
                    bh = b.cpu()
                    dist.all_reduce(bh, op=dist.ReduceOp.SUM, group=self.group)
                    b.copy_(bh)
                torch.cuda.synchronize(self.device)
                return 0
            except Exception as e:
                self.errors.append(e)
                return -1

        self._ag = _lib.GG_ALLGATHER_FN(allgather)
        self._ar = _lib.GG_ALLREDUCE_I32_FN(allreduce_i32)

    def struct(self):
        from . import _lib
        return _lib.gg_collective(self.rank, self.world, self._ag, self._ar, None)
