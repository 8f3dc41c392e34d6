"""Batch partitioning across ranks (one process per GPU).

The solve is embarrassingly parallel over systems (the
XGC proxy app is "parallelized over spatial mesh nodes and is embarrassingly
parallel"), so there is NO collective on the solve path: every rank solves
its own contiguous slice of global system indices.  torch.distributed is
used only for plumbing around the timed region: a barrier, the max of the
per-rank device times, and one gather of the per-system convergence stats.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Slice:
    rank: int
    world: int
    g0: int        # first global system index of this rank
    count: int     # systems on this rank
    total: int     # systems over all ranks


def rank_slice(batch: int, rank: int, world: int, scaling: str = "weak") -> Slice:
    """Contiguous slice of global indices for `rank`.

    weak:   every rank solves `batch` systems; global indices
            [rank*batch, (rank+1)*batch)  (work per GPU fixed as N grows).
    strong: `batch` systems in total split as evenly as possible; the first
            batch % world ranks get one more.  Ion/electron interleave by
            global index parity, so every slice stays ~50/50.
    """
    if world < 1 or not 0 <= rank < world:
        raise ValueError(f"bad rank {rank} / world {world}")
    if batch < 0:
        raise ValueError("batch must be >= 0")
    if scaling == "weak":
        return Slice(rank, world, rank * batch, batch, batch * world)
    if scaling != "strong":
        raise ValueError(f"scaling must be weak or strong, not {scaling!r}")
    base, extra = divmod(batch, world)
    g0 = rank * base + min(rank, extra)
    return Slice(rank, world, g0, base + (1 if rank < extra else 0), batch)


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank scalar (e.g. elapsed ms) over the default group."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_stats(iters, resnorm, status):
    """All-gather per-system (iters, resnorm, status) of every rank, in rank
    (= global-index) order.  Slices may differ in length (strong scaling), so
    each rank pads to the longest one.  The tensors' device must suit the
    backend (CUDA for NCCL, CPU for gloo).  Returns CPU tensors."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return iters.cpu(), resnorm.cpu(), status.cpu()
    world = dist.get_world_size()
    cnt = torch.tensor([iters.numel()], dtype=torch.int64, device=iters.device)
    cnts = [torch.empty_like(cnt) for _ in range(world)]
    dist.all_gather(cnts, cnt)
    counts = [int(c.item()) for c in cnts]
    mx = max(counts)
    outs = []
    for t in (iters, resnorm, status):
        pad = torch.zeros(mx, dtype=t.dtype, device=t.device)
        pad[: t.numel()] = t
        bufs = [torch.empty_like(pad) for _ in range(world)]
        dist.all_gather(bufs, pad)
        outs.append(torch.cat([b[:c] for b, c in zip(bufs, counts)]).cpu())
    return tuple(outs)
