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


class ShardExecutor:
    """One global batch per step with its rows sharded over the ranks (SURVEY.md §8(e) item 1,
    strong scaling): rank 0 holds the step's inputs, every input is scattered in contiguous row
    blocks (one collective per input), each rank runs `runner(shard_inputs, shard_outputs)` on
    its rows, and every output is gathered back to rank 0 in rank order.  Rows are independent
    (BN folded; the only cross-row operators are per-row joins), so the result equals the
    single-GPU run of the whole batch.  With NCCL everything is enqueued on the current stream
    (no host synchronisation inside a step); with gloo device tensors are staged through host
    memory (the one-GPU test of the multi-rank flow).

    in_meta / out_meta: [(trailing shape, torch dtype)] per input / output; n_rows must divide by
    the world size (NCCL scatter/gather move equal blocks)."""

    def __init__(self, n_rows: int, in_meta, out_meta, device: torch.device):
        self.world = dist.get_world_size() if dist.is_initialized() else 1
        self.rank = dist.get_rank() if dist.is_initialized() else 0
        if n_rows % self.world:
            raise ValueError(f"batch {n_rows} does not split evenly over {self.world} ranks")
        self.n_rows, self.rows = n_rows, n_rows // self.world
        self.device = device
        self.staged = dist.is_initialized() and dist.get_backend() == "gloo" and device.type == "cuda"
        mk = lambda shape, dt: torch.empty((self.rows,) + tuple(shape), dtype=dt, device=device)  # noqa: E731
        self.shard_in = [mk(s, d) for s, d in in_meta]
        self.shard_out = [mk(s, d) for s, d in out_meta]
        self.out_meta = out_meta

    def bytes_moved(self):
        """(scatter bytes leaving rank 0, gather bytes arriving at rank 0) per step."""
        ob = (self.world - 1) * self.rows
        sc = sum(t[0].numel() * t.element_size() * ob for t in self.shard_in)
        ga = sum(t[0].numel() * t.element_size() * ob for t in self.shard_out)
        return sc, ga

    def _scatter(self, full, shard):
        if self.world == 1:
            shard.copy_(full)
            return
        if self.staged:
            tmp = torch.empty(shard.shape, dtype=shard.dtype)
            chunks = list(full.cpu().chunk(self.world)) if self.rank == 0 else None
            dist.scatter(tmp, chunks, src=0)
            shard.copy_(tmp)
            return
        dist.scatter(shard, list(full.chunk(self.world)) if self.rank == 0 else None, src=0)

    def _gather(self, shard, full):
        if self.world == 1:
            full.copy_(shard)
            return
        if self.staged:
            bufs = [torch.empty(shard.shape, dtype=shard.dtype) for _ in range(self.world)] if self.rank == 0 else None
            dist.gather(shard.cpu(), bufs, dst=0)
            if self.rank == 0:
                full.copy_(torch.cat(bufs))
            return
        dist.gather(shard, list(full.chunk(self.world)) if self.rank == 0 else None, dst=0)

    def step(self, inputs, outputs, runner):
        """inputs / outputs: full-batch tensors on rank 0 (ignored elsewhere).  runner(shard_in,
        shard_out) computes this rank's rows in place."""
        for i, s in enumerate(self.shard_in):
            self._scatter(inputs[i] if self.rank == 0 else None, s)
        runner(self.shard_in, self.shard_out)
        for i, s in enumerate(self.shard_out):
            self._gather(s, outputs[i] if self.rank == 0 else None)


def calibrate_link(sizes=(1 << 12, 1 << 16, 1 << 20, 1 << 24), reps: int = 20, peer: int = 1):
    """Measured NVLink cut-edge cost for the comm model (§III-B, Fig. 5: transfer
    latency is linear in the message size): rank 0 <-> `peer` NCCL send/recv ping-pong per size,
    timed with CUDA events on rank 0; one-way time = half the round trip.  A least-squares line
    t = alpha + bytes * ps_per_byte / 1000 gives the comm model's cross-GPU link (integer ns and
    ps per byte, include/duet.h duet_link).  Every rank must call it; returns the same dict on
    every rank, or None without a second GPU (single rank)."""
    if not dist.is_initialized() or dist.get_world_size() < 2 or dist.get_backend() != "nccl":
        return None
    rank = dist.get_rank()
    dev = torch.device("cuda", torch.cuda.current_device())
    pts = []
    for nb in sizes:
        buf = torch.empty(nb, dtype=torch.uint8, device=dev)
        ms = None
        for it in range(reps + 3):
            if rank == 0:
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                dist.send(buf, peer)
                dist.recv(buf, peer)
                e1.record()
                e1.synchronize()
                if it >= 3:
                    t = e0.elapsed_time(e1) / 2
                    ms = t if ms is None else min(ms, t)
            elif rank == peer:
                dist.recv(buf, 0)
                dist.send(buf, 0)
        if rank == 0:
            pts.append((nb, ms * 1e6))
    res = [None]
    if rank == 0:
        xs = [p[0] for p in pts]
        ys = [p[1] for p in pts]
        n = len(xs)
        mx, my = sum(xs) / n, sum(ys) / n
        slope = sum((x - mx) * (y - my) for x, y in zip(xs, ys)) / max(sum((x - mx) ** 2 for x in xs), 1e-30)
        alpha = my - slope * mx
        res[0] = {"alpha_ns": max(0, int(round(alpha))), "ps_per_byte": max(0, int(round(slope * 1000))),
                  "points_ns": [(int(b), round(t, 1)) for b, t in pts], "peer": peer}
    dist.broadcast_object_list(res, src=0)
    return res[0]
