"""C5: the corpus shard loop bench.py runs per rank, driven here for
G in {1, 2, 4} virtual ranks on one GPU.  Contiguous clip ranges (shard_clips), one
pipeline call per clip with the clip's global frame base, per-clip device counters:
the per-clip window hashes, the totals and the corpus digest are identical for every G
(clips never interact on this path)."""
import pytest
import torch

from synth import configs, video, weights
from tests.helpers import threshold

pytestmark = pytest.mark.gpu

otif = pytest.importorskip("paper_conf_sigmod_bastanim22_b200")
from paper_conf_sigmod_bastanim22_b200 import dist as odist  # noqa: E402


def test_c5_shard_loop_invariant_over_world_sizes():
    wl = configs.C5
    fpc, pool_clips, n_clips = 45, 4, 12
    pool = torch.empty((pool_clips * fpc, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
    for j in range(pool_clips):
        video.make_scene(wl, clip=j).render(range(fpc), out=pool[j * fpc:(j + 1) * fpc])
    pipe = otif.Pipeline(wl, weights.proxy_weights(), threshold("C2", 0.7), max_batch=fpc)

    def run_clip(k):
        j = k % pool_clips
        pipe.run_device(pool[j * fpc:(j + 1) * fpc], frame_base=k * fpc)
        c = pipe.counters()
        pipe.reset_counters()
        return c

    results = {}
    for world in (1, 2, 4):
        rows = [odist.run_corpus(odist.shard_clips(n_clips, world, r), run_clip) for r in range(world)]
        allc = torch.cat([r for r in rows if r.numel()]).cpu()
        results[world] = (allc, odist.corpus_digest(allc))
    ref_c, ref_d = results[1]
    assert ref_d["frames"] == n_clips * fpc and ref_d["clips"] == n_clips
    assert ref_d["windows"] >= n_clips * fpc          # at least one window per frame
    # clips that read the same pool slot differ only in their global frame base: the
    # hash keys windows by global frame, so their hashes differ while the counts agree
    assert int(ref_c[0, 4]) != int(ref_c[pool_clips, 4])
    assert torch.equal(ref_c[0, :4], ref_c[pool_clips, :4])
    for world in (2, 4):
        c, d = results[world]
        assert torch.equal(c, ref_c), world
        assert d == ref_d, world
    # the bench's grouped loop: one call per pool-contiguous run of clips (max_batch = pool x
    # clip), per-clip hashes / windows from the per-frame results: same per-clip hashes,
    # windows and frames, same column totals, same digest
    big = otif.Pipeline(wl, weights.proxy_weights(), threshold("C2", 0.7), max_batch=pool_clips * fpc,
                        pack_overlap=2)

    def run_group(r):
        j = r.start % pool_clips
        big.run_device(pool[j * fpc:(j + len(r)) * fpc], frame_base=r.start * fpc)
        tot = big.counters()
        big.reset_counters()
        fh, fc = big.frame_results(len(r) * fpc)
        rows = torch.zeros((len(r), tot.numel()), dtype=torch.int64, device=tot.device)
        rows[0] = tot
        rows[:, 0] = fpc
        rows[:, 2] = fc.view(len(r), fpc).sum(1)
        rows[:, 4] = fh.view(len(r), fpc).sum(1)
        return rows

    for world in (1, 2, 4):
        rows = [odist.run_corpus_grouped(odist.shard_clips(n_clips, world, r), pool_clips, run_group)
                for r in range(world)]
        big.flush()
        g = torch.cat([r for r in rows if r.numel()]).cpu()
        assert torch.equal(g[:, [0, 2, 4]], ref_c[:, [0, 2, 4]]), world
        assert torch.equal(g.sum(0), ref_c.sum(0)), world
        assert odist.corpus_digest(g) == ref_d, world
