#!/usr/bin/env python
"""§8(f) on the GPU: NEXT-1 window-size selection over ground-truth masks and the NEXT-2
proxy-tuning sweep (BASELINE.json configs[3]: proxy resolution x threshold x cell size on
1280x720 video), timed on the device.  Prints one JSON object.

    python scripts/sweep.py [--frames 450] [--k 3]
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sigmod_bastanim22_b200 import tuning  # noqa: E402
from scripts import train_proxy  # noqa: E402
from synth import configs, video, weights  # noqa: E402


def thresholds(name):
    d = json.load(open(os.path.join(ROOT, "tests", "golden", "thresholds.json")))
    return [d["workloads"][name][q]["B"] for q in ("0.5", "0.7", "0.8", "0.9")]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--frames", type=int, default=450)
    ap.add_argument("--k", type=int, default=3)
    ap.add_argument("--train-steps", type=int, default=400)
    ap.add_argument("--trained-thresholds", default="0.02,0.05,0.1,0.2,0.35,0.5,0.7,0.9")
    args = ap.parse_args()
    out = {}
    # NEXT-1 on C2-shaped ground truth (perfect proxy)
    wl = configs.C2
    sc = video.make_scene(wl)
    masks = np.stack([video.gt_mask(sc.gt_boxes(t), wl.src_w, wl.src_h, wl.cell) for t in range(args.frames)])
    cands = tuning.candidate_sizes(wl.src_w, wl.src_h, wl.cell)
    m = torch.from_numpy(masks).cuda()
    tuning.choose_window_sizes(m[:8], wl.src_w, wl.src_h, wl.cell, cands[:4], k=2)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    chosen, sums, idx = tuning.choose_window_sizes(m, wl.src_w, wl.src_h, wl.cell, cands, k=args.k)
    dt = time.perf_counter() - t0
    out["next1"] = {"workload": f"C2 ground-truth masks, {args.frames} frames", "candidates": len(cands),
                    "k": args.k, "chosen": chosen, "sum_est": sums, "seconds": dt,
                    "paper_context": "3 s to compute W on Caldot1 (P:L336, V100 + Xeon)"}
    # NEXT-2 sweep on C4 (1280x720)
    base = configs.C4_BASE
    frames = video.frames(base, args.frames).cuda()
    sc4 = video.make_scene(base)
    boxes = []
    for t in range(args.frames):
        boxes += [(t, x0, y0, x1, y1) for (x0, y0, x1, y1) in sc4.gt_boxes(t) if x0 < x1 and y0 < y1]
    boxes = torch.tensor(boxes, dtype=torch.int32, device="cuda").reshape(-1, 5)
    # random-init proxy (north_star): the frozen quantile thresholds
    bt = {s.name: thresholds(s.name) for s in configs.C4_SWEEP}
    t0 = time.perf_counter()
    rows = tuning.proxy_sweep(frames, boxes, configs.C4_SWEEP, bt, weights.proxy_weights())
    torch.cuda.synchronize()
    out["next2_random_init"] = {"workload": f"C4 1280x720, {args.frames} frames, 6 (r, c) settings x 4 quantile "
                                            "thresholds", "seconds": time.perf_counter() - t0, "rows": rows}
    # trained proxies (NEXT-3, "we train proxy models at several pre-determined
    # resolutions"): one per (r, c) setting, trained on frames [frames, frames + 1024) of
    # the same camera, swept over thresholds on the measured frames [0, frames)
    bts = [float(x) for x in args.trained_thresholds.split(",")]
    trained_rows, train_info = [], {}
    for s in configs.C4_SWEEP:
        tw, info = train_proxy.train_weights(s, steps=args.train_steps, batch=32, clip=0, start=args.frames)
        train_info[s.name] = {k: info[k] for k in ("steps", "ms_per_step", "loss", "train_frames")}
        trained_rows += tuning.proxy_sweep(frames, boxes, [s], {s.name: bts}, tw)
    torch.cuda.synchronize()
    out["next2_trained"] = {"workload": f"C4 1280x720, {args.frames} frames, 6 (r, c) settings x {len(bts)} "
                                        "thresholds, proxies trained per setting", "train": train_info,
                            "rows": trained_rows}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
