"""Debug helper: run stages individually at a given batch size with sync after each."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sigmod_bastanim22_b200 as otif
from synth import configs, video, weights
import json

wl = configs.C2
n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
blob = weights.proxy_weights()
b = json.load(open("tests/golden/thresholds.json"))["workloads"]["C2"]["0.7"]["B"]
src = torch.empty((n, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
video.make_scene(wl).render(range(n), out=src)
torch.cuda.synchronize(); print("render ok", flush=True)
img = otif.otif_resize(src, wl.proxy_h, wl.proxy_w); torch.cuda.synchronize(); print("resize ok", flush=True)
px = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, blob)
s = px.score(img); torch.cuda.synchronize(); print("proxy ok", s.mean().item(), flush=True)
r = otif.otif_select_windows(s, None, b, wl.src_w, wl.src_h, wl.cell, wl.sizes, want_mask=True)
torch.cuda.synchronize(); print("select ok", r["total"].item(), flush=True)
bt, slot, sc = otif.otif_pack_windows(src, wl.src_h, wl.src_w, r["windows"], r["total"], wl.sizes, [4 * n] * 3)
torch.cuda.synchronize(); print("pack ok", sc.tolist(), flush=True)
pipe = otif.Pipeline(wl, blob, b, max_batch=int(sys.argv[2]) if len(sys.argv) > 2 else 256)
pipe.run_device(src); torch.cuda.synchronize(); print("pipeline ok", pipe.counters().tolist(), flush=True)
