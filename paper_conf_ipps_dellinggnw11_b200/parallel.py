"""Multi-GPU plumbing for PHAST: sources are independent, so each
rank sweeps its own contiguous shard of them on its own replica of the hierarchy
(§V "assign different sources to each core"; §VIII-E "we
also copy the graph to each local memory bank explicitly").  The only collective
is the diameter's MAX all-reduce of one scalar (§VII-B "The maximum of
these values is the diameter").  torch.distributed is the transport (NCCL on GPUs,
gloo in the CPU tests); nothing here computes distances.
"""
from __future__ import annotations

import os


def shard(count: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous slice [lo, hi) of `count` sources for `rank`; sizes differ by <= 1."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    base, extra = divmod(count, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def share_hierarchy(build, load, path: str, rank: int, barrier):
    """Rank 0 builds (host CH, once) and saves; the others load after a barrier.
    build() -> handle with .save(path); load(path) -> handle."""
    if rank == 0:
        h = build()
        h.save(path)
    barrier()
    if rank != 0:
        h = load(path)
    barrier()
    if rank == 0 and os.path.exists(path):
        os.unlink(path)
    return h


def allreduce_max_u32(value: int, device=None) -> int:
    """MAX over ranks of a uint32 (carried in int64: uint32 collectives are not
    portable across backends)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([int(value)], dtype=torch.int64, device=device)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return int(t.item())


def diameter_distributed(h, sources, k_batch: int = 64) -> int:
    """Exact diameter over `sources` with this rank's shard on this rank's GPU, then
    one NCCL MAX all-reduce (the method's only exchange step)."""
    import numpy as np
    import torch
    import torch.distributed as dist
    world = dist.get_world_size() if dist.is_initialized() else 1
    rank = dist.get_rank() if dist.is_initialized() else 0
    lo, hi = shard(len(sources), world, rank)
    local = 0
    if hi > lo:
        out = torch.zeros(1, dtype=torch.int32, device="cuda")
        h.diameter_async(np.asarray(sources[lo:hi], np.uint32), k_batch, out)
        h.sync()
        local = int(out.cpu().numpy().view(np.uint32)[0])
    return allreduce_max_u32(local, device="cuda")


def combine_centrality(t, reach: bool):
    """Combine per-rank partial centrality over disjoint source shards, in place:
    betweenness (fp64) adds up over sources, reach (uint32 bits in int32, values
    < 2^31 never assumed) is a max -- carried as int64 so the unsigned order holds
    (R16/R17).  No-op without an initialised process group."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return t
    if not reach:
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return t
    wide = (t.to(torch.int64) & 0xFFFFFFFF)
    dist.all_reduce(wide, op=dist.ReduceOp.MAX)
    t.copy_(wide.to(torch.int32))
    return t
