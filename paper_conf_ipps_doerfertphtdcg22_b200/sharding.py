"""Multi-GPU plumbing of the hot path: one process per GPU, independent
lookups / iterations / sites sharded by contiguous ranges, tables replicated, and one
collective -- the checksum all-reduce -- over NCCL (gloo in CPU tests).

Lookup i draws its energy and material from fast_forward_LCG(seed, 2i), so any contiguous
partition gives bit-identical per-lookup results and an identical integer checksum.
"""
from __future__ import annotations


def shard(total: int, rank: int, world: int):
    """Strong scaling: rank r owns [r*total//world, (r+1)*total//world) -> (first, count)."""
    if world <= 0 or not 0 <= rank < world or total < 0:
        raise ValueError("bad shard arguments")
    a = total * rank // world
    b = total * (rank + 1) // world
    return a, b - a


def weak_shard(per_rank: int, rank: int):
    """Weak scaling: rank r owns its own batch [r*per_rank, (r+1)*per_rank)."""
    if per_rank < 0 or rank < 0:
        raise ValueError("bad shard arguments")
    return rank * per_rank, per_rank


def _reduce(t, op, group):
    """all_reduce in place; with the gloo backend a CUDA tensor is staged through the host
    (gloo is only used to exercise the N > 1 path on one GPU or on CPUs)."""
    import torch.distributed as dist
    if t.is_cuda and dist.get_backend(group) == "gloo":
        h = t.cpu()
        dist.all_reduce(h, op=op, group=group)
        t.copy_(h)
    else:
        dist.all_reduce(t, op=op, group=group)
    return t


def allreduce_u64_sum(t, group=None):
    """In-place u64 sum across ranks.  Collectives have no uint64 op, so the bits are
    all-reduced as int64: two's-complement addition wraps exactly like u64 mod 2^64."""
    import torch
    import torch.distributed as dist
    _reduce(t.view(torch.int64), dist.ReduceOp.SUM, group)
    return t


def allreduce_f64_sum(t, group=None):
    import torch.distributed as dist
    return _reduce(t, dist.ReduceOp.SUM, group)


def allreduce_max(value: float, device, group=None) -> float:
    """Max over ranks of a host float (the device-timed step time, max over ranks)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([value], dtype=torch.float64, device=device)
    _reduce(t, dist.ReduceOp.MAX, group)
    return float(t.item())


def pick_device_and_backend(local_rank: int, world: int, n_devices: int):
    """One process per GPU over NCCL; if there are more ranks than GPUs (only to exercise
    the multi-rank path on a single-GPU box) ranks share devices and talk over gloo."""
    if n_devices <= 0:
        raise RuntimeError("no CUDA device (there is no CPU fallback)")
    if world <= n_devices:
        return local_rank, "nccl", False
    return local_rank % n_devices, "gloo", True
