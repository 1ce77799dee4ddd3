#!/usr/bin/env python
"""NEXT-3 on the GPU: train the segmentation proxy on synthetic ground truth
at several proxy resolutions / cell sizes (the C4 sweep settings: "we train
proxy models at several pre-determined resolutions"), timed with CUDA events; then
score held-out frames with the trained model through the bf16 inference path and
report recall (R18) and windows per frame at a threshold, against the random-init proxy.
Prints one JSON object.

    python scripts/train_proxy.py [--steps 300] [--batch 32] [--settings C4b,C4e]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sigmod_bastanim22_b200 as otif  # noqa: E402
from paper_conf_sigmod_bastanim22_b200 import train, tuning  # noqa: E402
from synth import configs, video, weights  # noqa: E402


def boxes_for(wl, ts, clip):
    sc = video.make_scene(wl, clip=clip)
    out = []
    for i, t in enumerate(ts):
        out += [(i, *b) for b in sc.gt_boxes(t) if b[0] < b[2] and b[1] < b[3]]
    return np.array(out, np.int32).reshape(-1, 5)


def evaluate(wl, w, frames, boxes, threshold=0.5):
    img = otif.otif_resize(frames, wl.proxy_h, wl.proxy_w)
    sc = otif.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, w).score(img)
    r = otif.otif_select_windows(sc, None, threshold, wl.src_w, wl.src_h, wl.cell, wl.sizes)
    tot = int(r["total"].item())
    cov = tuning.window_recall(boxes, r["windows"], r["offsets"], r["counts"])
    win = r["windows"][:tot].cpu().numpy()
    area = float((win[:, 3].astype(np.int64) * win[:, 4]).sum()) / (frames.shape[0] * wl.src_w * wl.src_h) if tot else 0.0
    return {"recall": cov / max(boxes.shape[0], 1), "windows_per_frame": tot / frames.shape[0],
            "window_area_fraction": area}


def train_weights(wl, steps=300, batch=32, lr=1e-3, n_train=1024, clip=0, start=0):
    """Train one proxy on sampled frames [start, start + n_train) of clip `clip` of workload
    wl (one camera; frames with at least one detection; labels P:L139; BCE + Adam,
    readings R26/R27) from the random init.
    -> (trained fp32 weight blob, info dict with the loss curve and ms per step)."""
    rng = np.random.default_rng(wl.seed + 7919 * clip + start)
    sc = video.make_scene(wl, clip=clip)
    cand = [i for i, t in enumerate(range(start, start + n_train)) if len(sc.gt_boxes(t)) > 0]
    frames = video.frames(wl, n_train, start=start, device="cuda", clip=clip)
    img_all = otif.otif_resize(frames, wl.proxy_h, wl.proxy_w)
    del frames
    gh, gw = -(-wl.src_h // wl.cell), -(-wl.src_w // wl.cell)
    lab_all = train.otif_cell_labels(torch.from_numpy(boxes_for(wl, range(start, start + n_train), clip)).cuda(),
                                     n_train, (gh, gw), wl.src_w, wl.src_h, wl.cell)
    cand_t = torch.tensor(cand, device="cuda")
    w0 = weights.proxy_weights()
    tr = train.Trainer(wl.proxy_h, wl.proxy_w, wl.n_strided, w0, max_batch=batch)
    order = [cand_t[torch.from_numpy(rng.choice(len(cand), batch, replace=False)).cuda()] for _ in range(steps)]
    losses = []
    tr.step(img_all[order[0]], lab_all[order[0]], lr)      # warm-up (not timed)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for s in range(1, steps):
        idx = order[s]
        loss = tr.step(img_all[idx], lab_all[idx], lr)
        if s % 25 == 0 or s == steps - 1:
            losses.append((s, loss.clone()))
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / max(steps - 1, 1)
    w = tr.weights()
    del tr, img_all, lab_all
    torch.cuda.empty_cache()
    info = {"setting": wl.name, "proxy": f"{wl.proxy_w}x{wl.proxy_h}", "cell": wl.cell, "batch": batch,
            "steps": steps, "train_clip": clip, "train_frames": [start, start + n_train], "ms_per_step": ms, "train_frames_per_s": batch / (ms / 1e3),
            "loss": [(s, float(l.item())) for s, l in losses]}
    return w, info


def run(settings, steps, batch, lr=1e-3, n_train=1024, n_eval=128):
    out = []
    for wl in settings:
        w, info = train_weights(wl, steps, batch, lr, n_train, clip=0)
        # held-out evaluation: clip 1
        ev_frames = video.frames(wl, n_eval, device="cuda", clip=1)
        ev_boxes = torch.from_numpy(boxes_for(wl, range(n_eval), 1)).cuda()
        trained = evaluate(wl, w, ev_frames, ev_boxes)
        rand = evaluate(wl, weights.proxy_weights(), ev_frames, ev_boxes)
        info["held_out_threshold_0.5"] = {"trained": trained, "random_init": rand}
        out.append(info)
        torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--batch", type=int, default=32)
    ap.add_argument("--settings", default=",".join(w.name for w in configs.C4_SWEEP))
    args = ap.parse_args()
    names = args.settings.split(",")
    settings = [w for w in configs.C4_SWEEP if w.name in names]
    print(json.dumps({"next3": run(settings, args.steps, args.batch)}))


if __name__ == "__main__":
    main()
