"""Time one proxy pass (otif_proxy_score) on a workload's proxy shape: python scripts/proxy_time.py C4a [frames]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, weights
name = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 450
wl = {w.name: w for w in [configs.C1, configs.C2, configs.C3] + list(configs.C4_SWEEP)}[name]
img = torch.randint(0, 256, (n, wl.proxy_h, wl.proxy_w, 3), dtype=torch.uint8, device="cuda")
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights.proxy_weights())
for _ in range(3):
    px.score(img)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10):
    px.score(img)
e1.record()
torch.cuda.synchronize()
print(name, os.environ.get("OTIF_E12", "1"), "proxy ms", round(e0.elapsed_time(e1) / 10, 4))
