"""Time one proxy pass (C2, 4500 random proxy images) with CUDA events (trace builds: OTIF_E12_TRACE bits)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
wl = configs.C2
img = torch.randint(0, 256, (4500, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
for _ in range(3):
    s = px.score(img)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    s = px.score(img)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 10
print("proxy ms", round(ms, 3))
