#!/usr/bin/env python
"""NEXT-4 on the GPU: build the track index over S* (resample, DBSCAN, centres) and refine
the query tracks, C6 sizes, timed per call with CUDA events.  Prints one JSON object.

    python scripts/tracks_bench.py [--reps 5]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sigmod_bastanim22_b200 import refine  # noqa: E402
from synth import tracks  # noqa: E402


def timed(fn, reps, trials=3):
    """Mean time of `reps` back-to-back calls (CUDA events), median over `trials` blocks
    (the blocks differ by the SM clock the power controller settles on)."""
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(trials):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            r = fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / reps)
    return float(np.median(ts)), r


def run(wl, reps=5):
    sc = tracks.make(wl)
    pts, off = sc.training(wl.n_train, wl.seed + 1)
    q, qo, ts, te, _ = sc.queries(wl.n_query, wl.gap, wl.seed + 2)
    pts, off, q, qo = [torch.from_numpy(a).cuda() for a in (pts, off, q, qo)]
    ws = torch.empty(int(refine.lib().otif_dbscan_workspace_bytes(wl.n_train)), dtype=torch.uint8, device="cuda")
    t_res, P = timed(lambda: refine.otif_track_resample(pts, off, wl.n_points), reps)
    t_db, (labels, core, nc) = timed(lambda: refine.otif_track_dbscan(P, wl.eps, wl.min_pts, workspace=ws), reps)
    n_clusters = int(nc.item())
    t_c, (C, sz) = timed(lambda: refine.otif_track_centers(P, labels, n_clusters), reps)
    t_ref, (out, used) = timed(lambda: refine.otif_track_refine(q, qo, C, sz, wl.k, wl.rho), reps)
    o = out.cpu().numpy()
    raw_s = q.cpu().numpy()[qo.cpu().numpy()[:-1]]
    raw_e = q.cpu().numpy()[qo.cpu().numpy()[1:] - 1]
    err_raw = float(np.hypot(*(raw_s - ts).T).mean() + np.hypot(*(raw_e - te).T).mean()) / 2
    err_ref = float(np.hypot(*(o[:, :2] - ts).T).mean() + np.hypot(*(o[:, 2:] - te).T).mean()) / 2
    pairs = wl.n_train * (wl.n_train + 1) / 2           # blocks on/above the diagonal ~ n^2/2
    return {"workload": f"{wl.name}: {wl.n_train} S* tracks (native rate), {wl.n_query} queries at g={wl.gap}, "
                        f"N={wl.n_points}, eps={wl.eps}, min_pts={wl.min_pts}, k={wl.k}, rho={wl.rho}",
            "timing": f"per call: median over 3 blocks of {reps} back-to-back calls (CUDA events)",
            "resample_ms": t_res, "dbscan_ms": t_db, "centers_ms": t_c, "refine_ms": t_ref,
            "index_build_ms": t_res + t_db + t_c, "refine_tracks_per_s": wl.n_query / (t_ref / 1e3),
            "clusters": n_clusters, "noise_fraction": float((labels < 0).float().mean().item()),
            "pair_distances_per_s": pairs / (t_db / 1e3), "refined_fraction": float((used > 0).float().mean().item()),
            "endpoint_error_px": {"raw": err_raw, "refined": err_ref}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    print(json.dumps(run(tracks.C6, args.reps)))


if __name__ == "__main__":
    main()
