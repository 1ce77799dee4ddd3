"""Multi-GPU plumbing: the path shards by video clip (frames never interact, P:L99
"one-minute clips"), so ranks need no data-path collective — only this bookkeeping and
one all_gather of per-rank int64 counters at the end."""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_clips(n_clips: int, world: int, rank: int) -> range:
    """Contiguous clip range of `rank` among `world` ranks: [r*n/G, (r+1)*n/G)."""
    if world <= 0 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    return range(rank * n_clips // world, (rank + 1) * n_clips // world)


def gather_counters(ctr: torch.Tensor, group=None) -> torch.Tensor:
    """int64 [C] per rank -> [world, C] on every rank (one all_gather_into_tensor on NCCL;
    all_gather on backends without it, e.g. gloo in the CPU tests)."""
    if not dist.is_available() or not dist.is_initialized():
        return ctr.view(1, -1).clone()
    world = dist.get_world_size(group)
    out = torch.empty((world, ctr.numel()), dtype=ctr.dtype, device=ctr.device)
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(out, ctr.view(1, -1).contiguous(), group=group)
    else:
        parts = list(out.unbind(0))
        dist.all_gather(parts, ctr.contiguous(), group=group)
        out = torch.stack(parts)
    return out


def combine(gathered: torch.Tensor) -> dict:
    """Totals over ranks; the window hash is a sum of 64-bit mixes, so it combines by
    wrapping addition and is independent of how clips were sharded."""
    tot = gathered.sum(0).tolist()
    return {"frames": tot[0], "positive_cells": tot[1], "windows": tot[2], "window_pixels": tot[3],
            "window_hash": int(tot[4]) & ((1 << 64) - 1), "per_size": tot[5:]}


def max_over_ranks(value: float, device="cpu") -> float:
    """Timing rule: the job time is the max over ranks."""
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
