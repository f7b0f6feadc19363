"""Host-side plumbing for one process per GPU (rank mode), over torch.distributed.

Control plane only — the data path (multisplit push, result pull) runs in the library's
kernels over NVLink peer memory.  Used by Table(rank=...):
  * allgather_bytes: exchange the ranks' exchange-arena handles (wd_rank_handle blobs);
  * allreduce_u64:   the host collective wd_rank_connect needs (batch-count agreement,
                     wd_size, barriers).
Both work on any backend (gloo on CPU for the tests, nccl on the GPU box).
"""
from __future__ import annotations

WD_REDUCE_SUM, WD_REDUCE_MAX = 0, 1


def _device_for(group=None):
    import torch
    import torch.distributed as dist
    backend = dist.get_backend(group)
    if backend == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def allgather_bytes(blob: bytes, group=None) -> list[bytes]:
    """Every rank's blob, in rank order."""
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, bytes(blob), group=group)
    return [bytes(b) for b in out]


def allreduce_u64(value: int, op: int, group=None) -> int:
    """Sum (op 0) or max (op 1) of one non-negative integer < 2^63 over the group."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([int(value)], dtype=torch.int64, device=_device_for(group))
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == WD_REDUCE_MAX else dist.ReduceOp.SUM,
                    group=group)
    return int(t.item())


def max_over_ranks(x: float, group=None) -> float:
    """Timing helper: the max of a float over the group (bench.py)."""
    import torch
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=_device_for(group))
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())
