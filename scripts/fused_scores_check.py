"""Fused-resize pipeline scores vs the stage path on small batches (a quick check on a GPU box: max |diff| must be 0)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights
blob = weights.proxy_weights()
for name, n in [(a.split(":")[0], int(a.split(":")[1])) for a in (sys.argv[1:] or ["C1:8", "C2:4"])]:
    wl = getattr(configs, name)
    src = video.frames(wl, n).cuda()
    pipe = otif.Pipeline(wl, blob, 0.5, max_batch=n)
    pipe.run_device(src)
    torch.cuda.synchronize()
    got = pipe.scores(n)
    img = otif.otif_resize(src, wl.proxy_h, wl.proxy_w)
    ref = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, blob).score(img)
    d = (got - ref).abs()
    print(name, n, "fused", pipe.resize_fused(), "max diff", d.max().item(), "frac diff", (d > 0).float().mean().item(), flush=True)
