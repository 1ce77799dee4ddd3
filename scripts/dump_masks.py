"""Dump the random-init proxy's cell masks at the bench threshold (q = 0.7) for a workload,
for offline component statistics of the grouping stage (gpurun_out/masks_<wl>.npz)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights
from tests.helpers import threshold
for name in sys.argv[1:] or ["C4b", "C3"]:
    wl = getattr(configs, name, None) or {w.name: w for w in configs.C4_SWEEP}[name]
    n = min(wl.n_frames, 450)
    src = video.frames(wl, n).cuda()
    b = threshold(wl.name, 0.7)
    pipe = otif.Pipeline(wl, weights.proxy_weights(), b, max_batch=n)
    pipe.run_device(src)
    torch.cuda.synchronize()
    sc = pipe.scores(n)
    r = otif.otif_select_windows(sc, None, b, wl.src_w, wl.src_h, wl.cell, wl.sizes, want_mask=True)
    np.savez_compressed(f"gpurun_out/masks_{name}.npz", mask=r["mask"].cpu().numpy())
    print(name, n, "positive", float(r["mask"].float().mean()))
