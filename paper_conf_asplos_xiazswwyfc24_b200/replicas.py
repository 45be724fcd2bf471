"""Multi-GPU plumbing for batch-sharded replicas (BASELINE.json north_star (c)).

Batch-1 inference of one request does not shard (PAPER.md is single-GPU), so N GPUs run N
independent replicas: each rank owns a contiguous shard of the request stream, runs it through its own
plan with no collective on the hot path, and torch.distributed is used only around the timed region
(barrier, max-over-ranks time) and afterwards (gathering outputs to rank 0 for the oracle check).
Backend-agnostic: NCCL over NVLink on the GPU box, gloo in the CPU tests.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def world():
    if dist.is_available() and dist.is_initialized():
        return dist.get_world_size(), dist.get_rank()
    return 1, 0


def shard(n_requests: int, world_size: int, rank: int) -> range:
    """Contiguous shard of request ids [0, n_requests) for `rank`; sizes differ by at most one."""
    base, extra = divmod(n_requests, world_size)
    lo = rank * base + min(rank, extra)
    return range(lo, lo + base + (1 if rank < extra else 0))


def max_over_ranks(x: float, device=None) -> float:
    """The job's time is the slowest rank's (timed on the device, reduced here)."""
    ws, _ = world()
    if ws == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def aggregate_rate(units_per_rank: int, max_seconds: float) -> float:
    """Whole-job throughput: units processed by all ranks / the slowest rank's time (weak scaling)."""
    ws, _ = world()
    return ws * units_per_rank / max_seconds


def gather_to_rank0(t: torch.Tensor):
    """Every rank's output (shape [n_r, ...], n_r may differ by rank: uneven request shards) on
    rank 0 as ONE tensor [sum n_r, ...] in rank order (for the parity check after timing); None
    elsewhere.  Shards are padded to the largest n_r for the collective and trimmed afterwards."""
    ws, rank = world()
    if ws == 1:
        return t
    dev = t.device
    n = torch.tensor([t.shape[0]], dtype=torch.int64, device=dev)
    ns = [torch.zeros_like(n) for _ in range(ws)]
    dist.all_gather(ns, n)
    sizes = [int(x.item()) for x in ns]
    mx = max(sizes)
    pad = torch.zeros((mx,) + tuple(t.shape[1:]), dtype=t.dtype, device=dev)
    pad[: t.shape[0]] = t
    parts = [torch.empty_like(pad) for _ in range(ws)]
    dist.all_gather(parts, pad)
    if rank != 0:
        return None
    return torch.cat([p[:k] for p, k in zip(parts, sizes)])
