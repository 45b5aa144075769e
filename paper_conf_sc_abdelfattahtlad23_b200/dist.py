"""Multi-GPU plumbing for the batched band solver.

The matrices of a batch are independent: there is no exchange step, so the
data path has no collective.  Rank r of R owns the contiguous shard
[floor(r*B/R), floor((r+1)*B/R)) of the global batch and generates it locally
from the counter-based generator (no scatter).  torch.distributed is used only
off the hot path: a barrier before timing, a MAX all-reduce of per-rank
device times (the reported time is the slowest rank), and an all-gather of
small verification summaries.
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist

from .inputs import shard_range

__all__ = ["shard_range", "env_rank", "init", "max_over_ranks", "gather_summaries"]


def env_rank() -> tuple[int, int, int]:
    """(rank, world, local_rank) from the torchrun environment (defaults: single process)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def init(backend: str | None = None) -> tuple[int, int, torch.device]:
    """Initialise the process group when WORLD_SIZE > 1; returns (rank, world, device)."""
    rank, world, local = env_rank()
    if backend is None:
        backend = "nccl" if torch.cuda.is_available() else "gloo"
    if backend == "nccl":
        torch.cuda.set_device(local)
        dev = torch.device("cuda", local)
    else:
        dev = torch.device("cpu")
    if world > 1 and not dist.is_initialized():
        kw = {"device_id": dev} if backend == "nccl" else {}
        dist.init_process_group(backend, **kw)
    return rank, world, dev


def max_over_ranks(values: list[float], device: torch.device) -> list[float]:
    """Element-wise MAX of per-rank values (device times) over all ranks."""
    t = torch.tensor(values, dtype=torch.float64, device=device)
    if dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.tolist()


def gather_summaries(summary: list[float], device: torch.device) -> list[list[float]]:
    """All-gather a fixed-length per-rank summary vector (e.g. checksums, info counts)."""
    t = torch.tensor(summary, dtype=torch.float64, device=device)
    if not (dist.is_initialized() and dist.get_world_size() > 1):
        return [t.tolist()]
    out = [torch.empty_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(out, t)
    return [o.tolist() for o in out]
