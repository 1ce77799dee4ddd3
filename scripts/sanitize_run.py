#!/usr/bin/env python
"""Small C1 run of every hot-path kernel for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): resize (even-factor and general), proxy (E1+E2 fused reading the
proxy image or the frames, several tiles per CTA, E3..D1 and
the S = 2 separate-E1 path), select (scores and mask input, 4- and 8-connectivity, the
deferred pass and the rescan path), pack (bulk, funnel and byte branches), the native
pipeline, NEXT-1 choose (multi-candidate launch) and the recall kernel.

    compute-sanitizer --tool racecheck python scripts/sanitize_run.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sigmod_bastanim22_b200 as otif  # noqa: E402
from paper_conf_sigmod_bastanim22_b200 import tuning  # noqa: E402
from synth import configs, masks, video, weights  # noqa: E402

wl = configs.C1
blob = weights.proxy_weights()
src = video.frames(wl, 4).cuda()
img = otif.otif_resize(src, wl.proxy_h, wl.proxy_w)
otif.otif_resize(src, 187, 333)
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, blob)
sc = px.score(img)
# a 640-wide proxy (E2 pitch 161: the slab overlap is longer than a tile and moved between
# the two slabs after a converter barrier), 8 frames = several tiles per CTA
c4d = configs.C4_SWEEP[3]
src_w = video.frames(c4d, 8).cuda()
img_w = otif.otif_resize(src_w, c4d.proxy_h, c4d.proxy_w)
otif.Proxy(c4d.proxy_h, c4d.proxy_w, c4d.n_strided, blob).score(img_w)
# an odd-width proxy image (105 px: 315-B rows, not 4-B aligned): the tile E1+E2 kernel
# (e12_umma_kernel) instead of e12s
c1o = wl.with_(name="C1o", src_w=420, sizes=((64, 64), (128, 128), (420, 256)))
img_o = otif.otif_resize(video.frames(c1o, 4).cuda(), c1o.proxy_h, c1o.proxy_w)
otif.Proxy(c1o.proxy_h, c1o.proxy_w, c1o.n_strided, blob).score(img_o)
s2 = wl.with_(name="C1s2", cell=8)
otif.Proxy(s2.proxy_h, s2.proxy_w, s2.n_strided, blob).score(img[:2])
r = otif.otif_select_windows(sc, None, 0.5, wl.src_w, wl.src_h, wl.cell, wl.sizes, want_mask=True)
rng = np.random.default_rng(0)
c4 = configs.C4_SWEEP[0]
m = np.concatenate([masks.sparse(rng, 8, 23, 40), masks.lattice(rng, 4, 23, 40)])
for conn in (4, 8):
    otif.otif_select_windows(None, torch.from_numpy(m).cuda(), 0.0, c4.src_w, c4.src_h, c4.cell,
                             [(32, 32, 2), (96, 32, 3), (c4.src_w, c4.src_h, 1000)], connectivity=conn)
    otif.otif_select_windows(None, torch.from_numpy(m).cuda(), 0.0, c4.src_w, c4.src_h, c4.cell,
                             [(s[0], s[1], s[0] * s[1] << 20) for s in c4.sizes], connectivity=conn)
rows = [(0, 0, 0, 64, 64, 0), (1, 5, 7, 64, 64, 0), (2, 16, 32, 128, 128, 1), (3, 0, 0, 416, 256, 2),
        (0, 300, 190, 100, 60, 3)]
wt = torch.tensor(rows, dtype=torch.int32, device="cuda")
otif.otif_pack_windows(src, wl.src_h, wl.src_w, wt, torch.tensor([len(rows)], dtype=torch.int32, device="cuda"),
                       list(wl.sizes) + [(100, 60)], [2, 1, 1, 1])
otif.otif_pack_windows(src, wl.src_h, wl.src_w, r["windows"], r["total"], wl.sizes, [8, 8, 4])
pipe = otif.Pipeline(wl, blob, 0.5, max_batch=3)
pipe.run_host(src.cpu().contiguous())
# resize fused into E1+E2 with several tiles per CTA (the slab overlap carried between tiles)
src_many = video.frames(wl, 170).cuda()
pipe_many = otif.Pipeline(wl, blob, 0.5, max_batch=170, pack_overlap=2)
pipe_many.run_device(src_many)
pipe_many.flush()
assert pipe_many.resize_fused()
gm = torch.from_numpy(np.stack([video.gt_mask(video.make_scene(wl).gt_boxes(t), wl.src_w, wl.src_h, wl.cell)
                                for t in range(4)])).cuda()
tuning.choose_window_sizes(gm, wl.src_w, wl.src_h, wl.cell, tuning.candidate_sizes(wl.src_w, wl.src_h, wl.cell)[:6], k=3)
boxes = torch.tensor([[0, 10, 10, 50, 50], [1, 0, 0, 30, 20]], dtype=torch.int32, device="cuda")
tuning.window_recall(boxes, r["windows"], r["offsets"], r["counts"])
torch.cuda.synchronize()
print("sanitize run ok")
