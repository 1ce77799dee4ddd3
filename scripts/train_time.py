"""Time / profile target: one NEXT-3 training step (C2 proxy resolution, batch 32)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_sigmod_bastanim22_b200 import train as otif_train
from synth import configs, weights
wl = configs.C2
n = 32
img = torch.randint(0, 256, (n, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
lab = (torch.rand((n, gh, gw), device="cuda") < 0.3).to(torch.uint8)
tr = otif_train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights(), max_batch=n)
for _ in range(3):
    tr.step(img, lab, 1e-3)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    tr.step(img, lab, 1e-3)
e1.record()
torch.cuda.synchronize()
print("train step ms", e0.elapsed_time(e1) / 10)
