"""Seeded synthetic video for the OTIF hot path (recipe: DESIGN.md §5).

Traffic scene (fixed camera, 6 of the paper's 7 datasets): static textured
background with 2–3 straight road bands, solid-colour rectangles ("vehicles") with a
2-px half-intensity border that spawn at band ends as a Poisson process and move
along the band, plus ±2 per-frame sensor noise.  UAV scene (moving camera):
a translating periodic background and 3–6 dense clusters of small objects.

The generator is shared input plumbing: it holds none of the method's arithmetic.
Object trajectories are drawn on the host with numpy PCG64; pixels are rendered with
integer-only torch ops, so CPU and CUDA rendering are bit-identical (the fp64
background is computed once on the host).  Ground truth = the object rectangles
and the cell mask "cell intersects a rectangle" (label rule P:L139; the perfect-proxy
assumption of P:L153).
"""
from __future__ import annotations

import math

import numpy as np
import torch

M32 = 0xFFFFFFFF


def _hash(*vals):
    """32-bit integer hash of int64 tensors/ints (wraps identically on CPU and CUDA)."""
    consts = (0x9E3779B1, 0x85EBCA77, 0xC2B2AE3D, 0x27D4EB2F)
    h = None
    for i, v in enumerate(vals):
        term = (v * consts[i % 4]) & M32
        h = term if h is None else (h ^ term)
    h = h ^ (h >> 15)
    h = (h * 0x2C1B3C6D) & M32
    h = h ^ (h >> 12)
    h = (h * 0x297A2D39) & M32
    h = h ^ (h >> 15)
    return h


def _texture(width: int, height: int, rng: np.random.Generator, cam: int) -> np.ndarray:
    """Static background, uint8 [H, W, 3] (fp64 sin/cos on the host, once)."""
    s = width / 960.0
    lam = rng.uniform(30, 120, size=3) * s
    phi = rng.uniform(0, 2 * math.pi, size=3)
    y = np.arange(height, dtype=np.float64)[:, None]
    x = np.arange(width, dtype=np.float64)[None, :]
    lum = (100 + 40 * np.sin(2 * math.pi * x / lam[0] + phi[0]) * np.cos(2 * math.pi * y / lam[1] + phi[1])
           + 20 * np.sin(2 * math.pi * (x + y) / lam[2] + phi[2]))
    yy = np.arange(height, dtype=np.int64)[:, None]
    xx = np.arange(width, dtype=np.int64)[None, :]
    noise = (_hash(np.int64(cam) + 7, yy, xx) % 49).astype(np.float64) - 24.0
    base = lum + noise
    tints = np.array([0.9, 1.0, 1.1])
    img = np.clip(np.floor(base[:, :, None] * tints[None, None, :] + 0.5), 0, 255).astype(np.uint8)
    return img


class TrafficScene:
    """Fixed camera over 2–3 straight roads; ~10 concurrent objects at 960x540."""

    def __init__(self, width: int, height: int, seed: int, mean_objects: float = 10.0):
        self.W, self.H, self.seed = width, height, seed
        rng = np.random.Generator(np.random.PCG64(seed))
        self.rng = rng
        bg = _texture(width, height, rng, seed)
        s = width / 960.0
        nb = int(rng.integers(2, 4))
        bw = max(height // 8, 4)
        self.bands = []
        for b in range(nb):
            horiz = bool(b % 2 == 0) if nb == 2 else bool(rng.integers(0, 2))
            if horiz:
                c = int(rng.integers(bw, height - bw))
            else:
                c = int(rng.integers(bw, width - bw))
            self.bands.append((horiz, c))
            yy = np.arange(height)[:, None]
            xx = np.arange(width)[None, :]
            grey = (110 + (_hash(np.int64(seed) + 101 + b, yy, xx) % 13).astype(np.int64) - 6).astype(np.uint8)
            if horiz:
                lo, hi = c - bw // 2, c - bw // 2 + bw
                bg[lo:hi, :, :] = grey[lo:hi, :, None]
            else:
                lo, hi = c - bw // 2, c - bw // 2 + bw
                bg[:, lo:hi, :] = grey[:, lo:hi, None]
        self.band_w = bw
        self.bg = bg
        self.scale = s
        # mean lifetime ≈ band length / mean speed; spawn rate keeps ~mean_objects alive
        mean_speed = 12.0 * s
        mean_len = np.mean([(width if h else height) for h, _ in self.bands]) + 92 * s
        self.rate = mean_objects / (mean_len / mean_speed)
        self._objects = []      # (spawn_t, x0, y0, w, h, vx, vy, color)
        self._simulated_to = None

    def _simulate(self, n_frames: int):
        if self._simulated_to is not None and self._simulated_to >= n_frames:
            return
        rng = np.random.Generator(np.random.PCG64(self.seed + 1))
        objs = []
        warm = int(2 * (max(self.W, self.H) / (4.0 * self.scale)))  # pre-roll so t=0 is populated
        for t in range(-warm, n_frames):
            k = rng.poisson(self.rate)
            for _ in range(k):
                bi = int(rng.integers(0, len(self.bands)))
                horiz, c = self.bands[bi]
                ow = rng.uniform(24, 160) * self.scale
                oh = ow * rng.uniform(0.5, 1.0)
                if not horiz:
                    ow, oh = oh, ow
                ow, oh = max(int(ow), 2), max(int(oh), 2)
                speed = rng.uniform(4, 20) * self.scale
                d = 1 if rng.integers(0, 2) else -1
                lane = rng.uniform(-0.25, 0.25) * self.band_w
                color = rng.integers(0, 256, size=3)
                if horiz:
                    x0 = -ow if d > 0 else self.W
                    y0 = c + lane - oh / 2
                    objs.append((t, float(x0), float(y0), ow, oh, d * speed, 0.0, color))
                else:
                    y0 = -oh if d > 0 else self.H
                    x0 = c + lane - ow / 2
                    objs.append((t, float(x0), float(y0), ow, oh, 0.0, d * speed, color))
        self._objects = objs
        self._simulated_to = n_frames

    def rects(self, t: int):
        """Visible objects at sampled frame t, in spawn order: [(x0,y0,x1,y1,color)] clipped."""
        out = []
        for (t0, x0, y0, w, h, vx, vy, color) in self._objects:
            if t0 > t:
                break
            dt = t - t0
            x = int(math.floor(x0 + vx * dt))
            y = int(math.floor(y0 + vy * dt))
            xa, ya, xb, yb = max(x, 0), max(y, 0), min(x + w, self.W), min(y + h, self.H)
            if xa < xb and ya < yb:
                out.append((x, y, x + w, y + h, color))
        return out

    def render(self, frames, device="cpu", out: torch.Tensor | None = None) -> torch.Tensor:
        frames = list(frames)
        self._simulate(max(frames) + 1 if frames else 0)
        if out is None:
            out = torch.empty((len(frames), self.H, self.W, 3), dtype=torch.uint8, device=device)
        bg = torch.from_numpy(self.bg).to(out.device)
        yy = torch.arange(self.H, device=out.device, dtype=torch.int64)[:, None]
        xx = torch.arange(self.W, device=out.device, dtype=torch.int64)[None, :]
        for i, t in enumerate(frames):
            f = bg.to(torch.int16).clone()
            for (x, y, x1, y1, color) in self.rects(t):
                _draw_box(f, x, y, x1, y1, color)
            noise = (_hash(torch.tensor(self.seed, device=out.device) + 3, torch.tensor(t, device=out.device),
                           yy, xx) % 5).to(torch.int16) - 2
            f += noise[:, :, None]
            out[i] = f.clamp_(0, 255).to(torch.uint8)
        return out

    def gt_boxes(self, t: int):
        self._simulate(t + 1)
        return [(max(x, 0), max(y, 0), min(x1, self.W), min(y1, self.H)) for (x, y, x1, y1, _) in self.rects(t)]


def _draw_box(f: torch.Tensor, x: int, y: int, x1: int, y1: int, color, border: int = 2):
    H, W = f.shape[0], f.shape[1]
    c = torch.tensor([int(v) for v in color], dtype=torch.int16, device=f.device)
    xa, ya, xb, yb = max(x, 0), max(y, 0), min(x1, W), min(y1, H)
    if xa >= xb or ya >= yb:
        return
    f[ya:yb, xa:xb] = c // 2
    ia, ja, ib, jb = max(x + border, 0), max(y + border, 0), min(x1 - border, W), min(y1 - border, H)
    if ia < ib and ja < jb:
        f[ja:jb, ia:ib] = c


class UAVScene:
    """Moving camera (1–3 px/frame translation) over 3–6 dense clusters of 20–60
    small (8–40 px) objects moving ≤ 3 px/frame ("UAV video")."""

    def __init__(self, width: int, height: int, seed: int):
        self.W, self.H, self.seed = width, height, seed
        rng = np.random.Generator(np.random.PCG64(seed))
        self.tex = _texture(2 * width, 2 * height, rng, seed)
        self.cam_v = rng.uniform(1, 3, size=2) * rng.choice([-1, 1], size=2)
        nc = int(rng.integers(3, 7))
        objs = []
        for _ in range(nc):
            cx, cy = rng.uniform(0, width), rng.uniform(0, height)
            cv = rng.uniform(-2.0, 2.0, size=2)
            rad = rng.uniform(60, 200) * width / 1920
            for _ in range(int(rng.integers(20, 61))):
                ow = int(rng.uniform(8, 40))
                oh = int(rng.uniform(8, 40))
                ox = cx + rng.normal(0, rad)
                oy = cy + rng.normal(0, rad)
                v = cv + rng.uniform(-0.5, 0.5, size=2)
                objs.append((ox, oy, ow, oh, v[0], v[1], rng.integers(0, 256, size=3)))
        self._objects = objs

    def rects(self, t: int):
        out = []
        mw, mh = self.W + 80, self.H + 80
        for (ox, oy, w, h, vx, vy, color) in self._objects:
            x = int(math.floor((ox + vx * t) % mw)) - 40
            y = int(math.floor((oy + vy * t) % mh)) - 40
            if max(x, 0) < min(x + w, self.W) and max(y, 0) < min(y + h, self.H):
                out.append((x, y, x + w, y + h, color))
        return out

    def render(self, frames, device="cpu", out: torch.Tensor | None = None) -> torch.Tensor:
        frames = list(frames)
        if out is None:
            out = torch.empty((len(frames), self.H, self.W, 3), dtype=torch.uint8, device=device)
        tex = torch.from_numpy(self.tex).to(out.device)
        th, tw = tex.shape[0], tex.shape[1]
        yy = torch.arange(self.H, device=out.device, dtype=torch.int64)
        xx = torch.arange(self.W, device=out.device, dtype=torch.int64)
        for i, t in enumerate(frames):
            oy = int(math.floor(self.cam_v[1] * t)) % th
            ox = int(math.floor(self.cam_v[0] * t)) % tw
            f = tex[(yy + oy) % th][:, (xx + ox) % tw].to(torch.int16)
            for (x, y, x1, y1, color) in self.rects(t):
                _draw_box(f, x, y, x1, y1, color, border=1)
            noise = (_hash(torch.tensor(self.seed, device=out.device) + 3, torch.tensor(t, device=out.device),
                           yy[:, None], xx[None, :]) % 5).to(torch.int16) - 2
            f += noise[:, :, None]
            out[i] = f.clamp_(0, 255).to(torch.uint8)
        return out

    def gt_boxes(self, t: int):
        return [(max(x, 0), max(y, 0), min(x1, self.W), min(y1, self.H)) for (x, y, x1, y1, _) in self.rects(t)]


def make_scene(workload, clip: int = 0):
    seed = workload.seed + clip
    if workload.scene == "uav":
        return UAVScene(workload.src_w, workload.src_h, seed)
    return TrafficScene(workload.src_w, workload.src_h, seed, mean_objects=getattr(workload, "objects", 10.0))


def gt_mask(boxes, frame_w: int, frame_h: int, cell: int) -> np.ndarray:
    """Cell (cy,cx) is 1 iff it intersects a box (P:L139 label rule), cells clipped to the frame."""
    gh, gw = -(-frame_h // cell), -(-frame_w // cell)
    m = np.zeros((gh, gw), np.uint8)
    for (x0, y0, x1, y1) in boxes:
        if x0 >= x1 or y0 >= y1:
            continue
        cx0, cy0 = x0 // cell, y0 // cell
        cx1, cy1 = -(-x1 // cell), -(-y1 // cell)
        m[cy0:cy1, cx0:cx1] = 1
    return m


def frames(workload, n: int | None = None, start: int = 0, device="cpu", clip: int = 0) -> torch.Tensor:
    """Sampled frames [start, start+n) of a workload's clip, u8 NHWC."""
    n = workload.n_frames if n is None else n
    return make_scene(workload, clip).render(range(start, start + n), device=device)
