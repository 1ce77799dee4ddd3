"""Multi-GPU plumbing: the path shards by video clip (frames never interact, P:L99
"one-minute clips"), so ranks need no data-path collective — only this bookkeeping and
one all_gather of per-rank int64 counters at the end."""
from __future__ import annotations

import hashlib
from typing import Callable

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
    out = {"frames": tot[0], "positive_cells": tot[1], "windows": tot[2], "window_pixels": tot[3],
           "window_hash": int(tot[4]) & ((1 << 64) - 1), "per_size": tot[5:13]}
    if len(tot) >= 15:   # pipeline counters: windows dropped for batch_cap, pixels packed
        out["dropped_windows"] = tot[13]
        out["packed_pixels"] = tot[14]
    return out


def max_over_ranks(value: float, device="cpu") -> float:
    """Timing rule: the job time is the max over ranks."""
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def run_corpus(clips: range, run_clip: Callable[[int], torch.Tensor]) -> torch.Tensor:
    """The shard loop: run_clip(k) processes clip k and returns its int64 counters [C]
    (device or host); -> [len(clips), C] in clip order."""
    rows = [run_clip(k) for k in clips]
    if not rows:
        return torch.zeros((0, 0), dtype=torch.int64)
    return torch.stack(rows)


def clip_groups(clips: range, pool: int) -> list:
    """Split a contiguous clip range into runs whose frames are contiguous in the frame pool
    (clip k reads pool slot k mod pool): each run is one pipeline call."""
    out, start = [], clips.start
    for k in clips:
        if k != start and k % pool == 0:
            out.append(range(start, k))
            start = k
    if len(clips):
        out.append(range(start, clips.stop))
    return out


def run_corpus_grouped(clips: range, pool: int, run_group: Callable[[range], torch.Tensor]) -> torch.Tensor:
    """The shard loop with one call per pool-contiguous run of clips: run_group(r) -> per-clip
    counters [len(r), C] (exact frames, windows and window hash per clip; the group's other
    totals attributed to its first clip, so column sums stay exact)."""
    rows = [run_group(r) for r in clip_groups(clips, pool)]
    if not rows:
        return torch.zeros((0, 0), dtype=torch.int64)
    return torch.cat(rows)


def gather_clip_counters(per_clip: torch.Tensor, n_clips: int, width: int, group=None) -> torch.Tensor:
    """Per-clip counters of every rank -> [n_clips, width] on every rank, in clip order.
    Ranks hold contiguous clip ranges (shard_clips), so the gathered blocks concatenate
    in rank order; shards are padded to ceil(n_clips / world) rows for one all_gather."""
    dev = per_clip.device if per_clip.numel() else torch.device("cpu")
    if not dist.is_available() or not dist.is_initialized():
        return per_clip.reshape(-1, width).clone()
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    mx = -(-n_clips // world)
    mine = torch.zeros((mx, width), dtype=torch.int64, device=dev)
    got = len(shard_clips(n_clips, world, rank))
    if got:
        mine[:got] = per_clip.reshape(got, width)
    flat = gather_counters(mine.reshape(-1), group)            # [world, mx * width]
    parts = [flat[r].reshape(mx, width)[:len(shard_clips(n_clips, world, r))] for r in range(world)]
    return torch.cat(parts)


def corpus_digest(clip_counters: torch.Tensor) -> dict:
    """Totals over the corpus plus a digest of the ordered per-clip window hashes: both are
    independent of how the clips were sharded (the check of SURVEY §8(e))."""
    c = clip_counters.cpu()
    tot = combine(c) if c.numel() else {}
    hashes = [int(h) & ((1 << 64) - 1) for h in c[:, 4].tolist()] if c.numel() else []
    tot["clips"] = len(hashes)
    tot["per_clip_hash_sha256"] = hashlib.sha256(b"".join(h.to_bytes(8, "little") for h in hashes)).hexdigest()
    return tot
