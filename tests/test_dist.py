"""Multi-process (gloo, world_size 2) checks of the N>1 host logic: clip sharding
partitions the corpus, counters gather to every rank, totals and the window hash are
independent of the sharding, the job time is the max over ranks."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sigmod_bastanim22_b200 import dist as odist


def test_shard_clips_partition():
    for n in (480, 7, 1, 0):
        for world in (1, 2, 3, 4, 8):
            got = [c for r in range(world) for c in odist.shard_clips(n, world, r)]
            assert got == list(range(n))
            sizes = [len(odist.shard_clips(n, world, r)) for r in range(world)]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        odist.shard_clips(10, 2, 2)


def _per_clip_counters(clip: int) -> torch.Tensor:
    # deterministic fake per-clip pipeline counters (otif.h layout, 15 int64: frames, pos,
    # windows, pixels, hash, 8 per-size, dropped, packed pixels) standing in for run_clip
    g = torch.Generator().manual_seed(clip)
    v = torch.randint(0, 1000, (15,), generator=g, dtype=torch.int64)
    v[0] = 450
    v[4] = (clip * 0x9E3779B97F4A7C15) & 0x7FFFFFFFFFFFFFFF
    return v


def _worker(rank, world, port, n_clips, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # the real shard loop (bench.py C5) with a CPU stand-in for the per-clip pipeline call
    clips = odist.shard_clips(n_clips, world, rank)
    per_clip = odist.run_corpus(clips, _per_clip_counters)
    ctr = per_clip.sum(0) if len(clips) else torch.zeros(15, dtype=torch.int64)
    g = odist.gather_counters(ctr)
    allc = odist.gather_clip_counters(per_clip, n_clips, 15)
    t = odist.max_over_ranks(float(rank + 1))
    out[rank] = (g.clone(), t, odist.combine(g), allc.clone(), odist.corpus_digest(allc))
    dist.barrier()
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world,n_clips", [(2, 10), (3, 10), (2, 1)])
def test_gloo_gather_and_sharding_invariance(world, n_clips):
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), n_clips, out), nprocs=world, join=True)
    ref_rows = torch.stack([_per_clip_counters(c) for c in range(n_clips)])
    ref = ref_rows.sum(0)
    single = odist.corpus_digest(odist.run_corpus(range(n_clips), _per_clip_counters))
    for r in range(world):
        g, t, tot, allc, digest = out[r]
        assert g.shape == (world, 15)
        assert torch.equal(g.sum(0), ref)
        assert t == float(world)              # max over ranks
        assert tot["frames"] == 450 * n_clips
        assert tot["window_hash"] == int(ref[4]) & ((1 << 64) - 1)
        assert torch.equal(allc, ref_rows)    # per-clip counters in clip order, every rank
        assert digest == single               # per-clip hashes + totals independent of the sharding
    assert odist.combine(ref.view(1, -1)) == out[0][2]


def test_clip_groups_follow_the_pool():
    for n, pool in ((480, 8), (10, 4), (7, 8), (0, 8)):
        for world in (1, 2, 3, 4, 8):
            for r in range(world):
                clips = odist.shard_clips(n, world, r)
                groups = odist.clip_groups(clips, pool)
                assert [k for g in groups for k in g] == list(clips)
                for g in groups:
                    assert len(g) <= pool and g.start // pool == (g.stop - 1) // pool
