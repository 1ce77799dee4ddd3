"""Profile target: one proxy pass over 1024 C2 frames (E1+E2 fused kernel is the ncu capture)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
wl = configs.C2
img = torch.randint(0, 256, (1024, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
for _ in range(2):
    s = px.score(img)
torch.cuda.synchronize()
