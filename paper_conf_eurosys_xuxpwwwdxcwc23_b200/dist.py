"""Batch-dimension data parallelism: one process per
GPU, contiguous batch shards, weights replicated, and one all-gather of the
chain outputs.  Every activation layout keeps N outermost, so a
shard is a contiguous slice of every physical tensor (zero-copy in / out).

Device-agnostic host logic: the same functions run on CUDA tensors with the
NCCL backend (bench.py under torchrun) and on CPU tensors with gloo (tests).
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def shard_range(N: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous [lo, hi) image range of `rank`; the first N % world ranks
    take one extra image."""
    base, extra = divmod(N, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def init_from_env(backend: str | None = None):
    """(world, rank, local_rank); initialises the process group if WORLD_SIZE > 1."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1 and not dist.is_initialized():
        if backend is None:
            backend = "nccl" if torch.cuda.is_available() else "gloo"
        if backend == "nccl":
            torch.cuda.set_device(local)
            dist.init_process_group(backend, device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    return world, rank, local


def gather_outputs(local: torch.Tensor, world: int, N: int | None = None) -> torch.Tensor:
    """All-gather per-rank outputs along dim 0 (the batch dim of the physical
    layout) into one tensor on every rank.  With N given, shards may be
    uneven (shard_range): each rank pads its shard to ceil(N / world) rows,
    and the padding rows are dropped after the gather."""
    if world == 1:
        return local
    if N is not None and N % world:
        per = -(-N // world)
        if local.shape[0] < per:
            pad = torch.zeros((per - local.shape[0],) + tuple(local.shape[1:]), dtype=local.dtype,
                              device=local.device)
            local = torch.cat([local, pad])
        full = gather_outputs(local, world)
        parts = [full[r * per: r * per + (shard_range(N, r, world)[1] - shard_range(N, r, world)[0])]
                 for r in range(world)]
        return torch.cat(parts)
    out = torch.empty((world * local.shape[0],) + tuple(local.shape[1:]), dtype=local.dtype,
                      device=local.device)
    if local.device.type == "cuda":
        dist.all_gather_into_tensor(out, local.contiguous())
    else:  # gloo: all_gather into a list
        parts = [torch.empty_like(local) for _ in range(world)]
        dist.all_gather(parts, local.contiguous())
        torch.cat(parts, out=out)
    return out


def max_over_ranks(x: float, world: int, device=None) -> float:
    """Max of a per-rank scalar (timings are reported as the slowest rank)."""
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sharded_forward(N: int, world: int, rank: int, run_shard) -> torch.Tensor:
    """Row a10: rank `rank` runs the whole chain on its contiguous image range
    (run_shard(lo, hi) -> that shard's output, N outermost in its physical
    layout, so the shard is a contiguous slice) and one all-gather assembles
    the full batch on every rank.  Images are independent (O8), so the result
    equals the unsharded chain's."""
    lo, hi = shard_range(N, rank, world)
    local = run_shard(lo, hi)
    return gather_outputs(local, world, N)
