"""Multi-GPU plumbing for bulk execution: the p instances are independent
(P:71), so they shard across ranks with no collective on the data
path.  One process per GPU (torchrun); each rank generates its own shard on
its own device from GLOBAL instance ids (so nothing is scattered), runs the
kernels, and the only collectives are off the timed path: a max-reduce of the
per-rank step time and one all-gather of the per-rank result checksums.
Works with the NCCL backend on GPUs and with gloo on CPU (tests).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def weak_range(p_per_rank: int, rank: int) -> tuple[int, int]:
    """Weak scaling: every rank owns p_per_rank instances, [rank*p, (rank+1)*p)."""
    return rank * p_per_rank, (rank + 1) * p_per_rank


def strong_range(p_total: int, rank: int, world: int) -> tuple[int, int]:
    """Strong scaling: p_total instances split into contiguous near-equal shards."""
    return p_total * rank // world, p_total * (rank + 1) // world


def _device_for(group=None) -> torch.device:
    backend = dist.get_backend(group) if dist.is_initialized() else "gloo"
    return torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")


def max_over_ranks(x: float, group=None) -> float:
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([x], dtype=torch.float64, device=_device_for(group))
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def gather_checksums(local: int, group=None) -> list[int]:
    """All-gather one uint64 per rank (sent as int64 bits)."""
    v = int(local) & (2 ** 64 - 1)
    signed = v - 2 ** 64 if v >= 2 ** 63 else v
    t = torch.tensor([signed], dtype=torch.int64, device=_device_for(group))
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return [v]
    out = [torch.zeros_like(t) for _ in range(dist.get_world_size(group))]
    dist.all_gather(out, t, group=group)
    return [int(o.item()) & (2 ** 64 - 1) for o in out]


def combine_checksums(parts: list[int]) -> int:
    """Shard checksums add mod 2^64 to the whole problem's checksum (bulkgen.checksum)."""
    return sum(parts) % 2 ** 64
