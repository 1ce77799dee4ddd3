#!/usr/bin/env python
"""Two C2 pipeline steps (4500 frames each) for ncu captures of the proxy kernels of the
second step, with the fused pack of the first step riding in them (pack_overlap 2) or not.

    ncu --set full -k regex:"conv_umma|e12s?_umma" -s 5 -c 5 python scripts/prof_conv.py [--overlap 2]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sigmod_bastanim22_b200 as otif  # noqa: E402
from synth import configs, video, weights  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--overlap", type=int, default=2)
a = ap.parse_args()
wl = configs.C2
n = wl.n_frames
src = torch.empty((n, wl.src_h, wl.src_w, 3), dtype=torch.uint8, device="cuda")
video.make_scene(wl).render(range(n), out=src)
thr = json.load(open(os.path.join(ROOT, "tests", "golden", "thresholds.json")))["workloads"]["C2"]["0.7"]["B"]
pipe = otif.Pipeline(wl, weights.proxy_weights(), thr, max_batch=n, pack_overlap=a.overlap)
for _ in range(2):
    pipe.run_device(src)
pipe.flush()
torch.cuda.synchronize()
print("ok")
