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
