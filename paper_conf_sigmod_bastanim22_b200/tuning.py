"""§8(f) NEXT rows on top of the C ABI: fixed window-size selection (NEXT-1)
and the proxy-module tuning sweep (NEXT-2).  Orchestration only: every
frame-level computation (resize, proxy, grouping, est sums, recall) runs in libotif."""
from __future__ import annotations

import ctypes
from typing import Sequence

import numpy as np
import torch

from . import api
from ._lib import GridDesc, check, lib


def candidate_sizes(frame_w: int, frame_h: int, cell: int, max_cells: int | None = None):
    """Window-size candidates: multiples of the cell size up to the frame (excluding the
    full frame itself, which is always in W), area cost."""
    out = []
    for h in range(cell, frame_h + 1, cell):
        for w in range(cell, frame_w + 1, cell):
            if (w, h) == (frame_w, frame_h):
                continue
            if max_cells is not None and (w // cell) * (h // cell) > max_cells:
                continue
            out.append((w, h, w * h))
    return out


def choose_window_sizes(masks: torch.Tensor, frame_w: int, frame_h: int, cell: int, candidates, k: int = 3,
                        full_cost: int | None = None, connectivity: int = 4, stream=None):
    """NEXT-1 greedy W selection over ground-truth masks [n, gh, gw] (device u8).
    -> (list of chosen sizes starting with the full frame, Σ est after each addition)."""
    api._require_cuda(masks)
    n, gh, gw = masks.shape
    m = len(candidates)
    full_cost = frame_w * frame_h if full_cost is None else int(full_cost)
    ws = torch.empty(int(lib().otif_choose_workspace_bytes(n, gh, gw, m)) + 256, dtype=torch.uint8, device=masks.device)
    g = GridDesc(frame_w, frame_h, cell, connectivity)
    idx = (ctypes.c_int32 * k)()
    est = (ctypes.c_int64 * k)()
    check(lib().otif_choose_window_sizes(api._ptr(masks), n, gh, gw, ctypes.byref(g), api.wsizes(candidates), m,
                                         full_cost, k, idx, est, api._ptr(ws), ws.numel(), api._stream(stream)),
          "otif_choose_window_sizes")
    chosen, sums = [], []
    for i in range(k):
        if idx[i] == -2:
            break
        chosen.append((frame_w, frame_h, full_cost) if idx[i] == -1 else tuple(candidates[idx[i]]))
        sums.append(int(est[i]))
    return chosen, sums, [int(idx[i]) for i in range(len(chosen))]


def window_recall(boxes: torch.Tensor, windows: torch.Tensor, offsets: torch.Tensor, counts: torch.Tensor,
                  stream=None) -> int:
    """NEXT-2 recall numerator: boxes int32 [nb, 5] (frame, x0, y0, x1, y1) on the device."""
    api._require_cuda(boxes, windows, offsets, counts)
    out = torch.zeros(1, dtype=torch.int64, device=boxes.device)
    check(lib().otif_window_recall(api._ptr(boxes), boxes.shape[0], api._ptr(windows), api._ptr(offsets),
                                   api._ptr(counts), counts.shape[0], api._ptr(out), api._stream(stream)),
          "otif_window_recall")
    return int(out.item())


def proxy_sweep(frames: torch.Tensor, boxes: torch.Tensor, workloads: Sequence, thresholds: dict, weights,
                sizes=None, connectivity: int = 4):
    """NEXT-2 caching + tuning phases: for each proxy resolution/cell setting i,
    run resize + proxy ONCE (timed with CUDA events -> T_proxy,i) and cache the scores;
    for each threshold B_j group the cells into windows and report the runtime estimate
    T_proxy,i + Σ_k T_{r_k.w, r_k.h} and the recall of the ground-truth boxes.
    frames: device u8 [n, H, W, 3]; boxes: device int32 [nb, 5]; thresholds: {name: [B_j]}.
    -> list of dict rows."""
    rows = []
    n = frames.shape[0]
    nb = boxes.shape[0]
    for wl in workloads:
        W = list(sizes) if sizes is not None else list(wl.sizes)
        px = api.Proxy(wl.proxy_h, wl.proxy_w, wl.n_strided, weights)
        img = api.otif_resize(frames, wl.proxy_h, wl.proxy_w)
        px.score(img)  # warm-up (workspace initialisation)
        times = []
        for _ in range(5):  # T_proxy,i: median of 5 device-timed resize + proxy passes
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            img = api.otif_resize(frames, wl.proxy_h, wl.proxy_w)
            scores = px.score(img)
            e1.record()
            torch.cuda.synchronize()
            times.append(e0.elapsed_time(e1))
        t_proxy_ms = sorted(times)[len(times) // 2]
        for b in thresholds[wl.name]:
            r = api.otif_select_windows(scores, None, b, wl.src_w, wl.src_h, wl.cell, W, connectivity=connectivity)
            total = int(r["total"].item())
            est = int(r["est_sum"].item())          # Σ_t est(R_t), summed by the grouping kernel
            cov = window_recall(boxes, r["windows"], r["offsets"], r["counts"])
            rows.append({"setting": wl.name, "proxy_w": wl.proxy_w, "proxy_h": wl.proxy_h, "cell": wl.cell,
                         "threshold": b, "t_proxy_ms": t_proxy_ms, "est_detector_cost": est, "windows": total,
                         "recall": cov / nb if nb else 1.0, "frames": n})
        px.close()
    return rows
