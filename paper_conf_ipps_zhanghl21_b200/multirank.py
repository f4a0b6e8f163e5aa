"""One-process-per-GPU plumbing for multi-GPU runs (torch.distributed; NCCL on GPUs, gloo on CPU).

DUET's data path shards by batch: inference rows are independent, so each
rank runs its own schedule on its own rows and no collective touches the data path.  Collectives
are used only for timing (max over ranks) and, when a caller wants one global result, to gather
row shards onto rank 0.
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def env():
    """(rank, world_size, local_rank) from the torchrun environment (defaults: single process).
    DUET_FORCE_DEVICE=<i> (test only) puts every rank on GPU i, so the multi-rank flow can run on a
    one-GPU box (with DUET_DIST_BACKEND=gloo: NCCL refuses two ranks on one GPU)."""
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("DUET_FORCE_DEVICE") is not None:
        local = int(os.environ["DUET_FORCE_DEVICE"])
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), local)


def init(backend: str | None = None, device: torch.device | None = None) -> bool:
    """Initialise the default process group when WORLD_SIZE > 1. Returns True if distributed."""
    rank, world, _ = env()
    if world <= 1 or dist.is_initialized():
        return dist.is_initialized()
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    backend = os.environ.get("DUET_DIST_BACKEND", backend)  # test override (see env())
    if backend is None:
        backend = "nccl" if torch.cuda.is_available() else "gloo"
    kw = {"device_id": device} if (backend == "nccl" and device is not None) else {}
    dist.init_process_group(backend, rank=rank, world_size=world, **kw)
    return True


def _dev():
    if dist.is_initialized() and dist.get_backend() == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def max_over_ranks(x: float) -> float:
    """The slowest rank's value (timing rule: a multi-GPU time is the max over ranks)."""
    if not dist.is_initialized():
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=_dev())
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def shard_range(n_rows: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous, near-equal row shard [start, stop) of rank `rank` (first n_rows % world ranks get
    one extra row)."""
    base, extra = divmod(n_rows, world)
    start = rank * base + min(rank, extra)
    return start, start + base + (1 if rank < extra else 0)


def gather_rows(local: torch.Tensor, n_rows: int) -> torch.Tensor | None:
    """Concatenate every rank's row shard (rank order) on rank 0; other ranks get None."""
    if not dist.is_initialized():
        return local
    world, rank = dist.get_world_size(), dist.get_rank()
    widest = max(shard_range(n_rows, world, r)[1] - shard_range(n_rows, world, r)[0] for r in range(world))
    pad = torch.zeros((widest,) + tuple(local.shape[1:]), dtype=local.dtype, device=_dev())
    pad[: local.shape[0]] = local.to(pad.device)
    bufs = [torch.empty_like(pad) for _ in range(world)] if rank == 0 else None
    dist.gather(pad, bufs, dst=0)
    if rank != 0:
        return None
    parts = []
    for r in range(world):
        a, b = shard_range(n_rows, world, r)
        parts.append(bufs[r][: b - a])
    return torch.cat(parts)


def barrier():
    if dist.is_initialized():
        dist.barrier()


def finalize():
    if dist.is_initialized():
        dist.destroy_process_group()
