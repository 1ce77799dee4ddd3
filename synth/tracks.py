"""Seeded synthetic object tracks for NEXT-4, track refinement (Fig. 4).

A fixed camera over a four-arm junction: every track follows one route (entry arm ->
exit arm, a quadratic Bezier through the junction, right-hand lanes), offset sideways
inside its lane, at a constant speed, with per-detection jitter.  One arm ends at a
"horizon" inside the frame and some tracks are cut short by occlusion ("tracks
may start or end at the horizon, or anywhere in the frame due to an occlusion").

* ``training(...)``  — S*: tracks at the native frame rate (θ_best).
* ``queries(...)``   — tracks captured at sampling gap g: every g-th detection from a
  random phase, so their first and last detections are offset from the true start and
  end; the true start/end are returned for the refinement-error statistic.

Output format (both): points float32 [total, 2] (x, y = box centres in pixels),
offsets int64 [n + 1] (track t is points[offsets[t]:offsets[t+1]]).  The generator is
input plumbing only: it holds none of the method's arithmetic (resampling, distances,
DBSCAN, medians live in oracle/ and in the CUDA library, independently).
"""
from __future__ import annotations

import dataclasses

import numpy as np


@dataclasses.dataclass(frozen=True)
class TrackWorkload:
    name: str
    width: int
    height: int
    n_train: int          # |S*|
    n_query: int
    gap: int              # sampling gap of the query tracks
    seed: int
    n_points: int = 20    # N ("In our implementation, N = 20")
    k: int = 10           # k nearest clusters ("k = 10")
    eps: float = 12.0     # DBSCAN radius in pixels (reading R23)
    min_pts: int = 8      # DBSCAN core threshold (reading R23)
    rho: float = 32.0     # "pass close to d1 and dn" radius in pixels (reading R24)


def _bezier(p0, p1, p2, m: int):
    t = np.linspace(0.0, 1.0, m)[:, None]
    return (1 - t) ** 2 * p0 + 2 * (1 - t) * t * p1 + t ** 2 * p2


class JunctionScene:
    """Four arms (N, E, S, W) meeting near the frame centre; 12 routes; route popularity
    from a Dirichlet draw, so some paths are rare ("infrequently-occurring paths")."""

    FINE = 1024   # samples of each route's base curve

    def __init__(self, width: int, height: int, seed: int):
        self.W, self.H = width, height
        rng = np.random.Generator(np.random.PCG64(seed))
        s = width / 1280.0
        self.scale = s
        self.lane = 14.0 * s
        cx = width * (0.5 + rng.uniform(-0.08, 0.08))
        cy = height * (0.5 + rng.uniform(-0.08, 0.08))
        self.centre = np.array([cx, cy])
        # arm end points on the border (N arm ends at a horizon inside the frame)
        ends = {
            "N": np.array([cx + rng.uniform(-0.1, 0.1) * width, height * rng.uniform(0.18, 0.3)]),
            "E": np.array([width - 1.0, cy + rng.uniform(-0.15, 0.15) * height]),
            "S": np.array([cx + rng.uniform(-0.1, 0.1) * width, height - 1.0]),
            "W": np.array([0.0, cy + rng.uniform(-0.15, 0.15) * height]),
        }
        arms = list(ends)
        self.routes = []
        for a in arms:
            for b in arms:
                if a == b:
                    continue
                p0, p2 = ends[a], ends[b]
                # right-hand traffic: shift the whole route to the right of its direction
                d = p2 - p0
                nrm = np.array([-d[1], d[0]]) / max(np.hypot(*d), 1e-9)
                shift = -1.5 * self.lane * nrm
                base = _bezier(p0 + shift, self.centre + shift * 0.5, p2 + shift, self.FINE)
                seg = np.hypot(*np.diff(base, axis=0).T)
                cum = np.concatenate([[0.0], np.cumsum(seg)])
                tang = np.gradient(base, axis=0)
                tang /= np.maximum(np.hypot(tang[:, 0], tang[:, 1]), 1e-12)[:, None]
                normal = np.stack([-tang[:, 1], tang[:, 0]], axis=1)
                self.routes.append((base, cum, normal))
        self.popularity = rng.dirichlet(np.full(len(self.routes), 0.8))

    def _draw(self, n: int, rng: np.random.Generator):
        """Continuous tracks: route, lateral offset, speed, start/end arc length."""
        route = rng.choice(len(self.routes), size=n, p=self.popularity)
        off = rng.uniform(-0.5, 0.5, size=n) * self.lane
        speed = rng.uniform(3.0, 10.0, size=n) * self.scale          # px per native frame
        length = np.array([self.routes[r][1][-1] for r in route])
        s0 = np.zeros(n)
        s1 = length.copy()
        occl = rng.uniform(size=n) < 0.15                              # occlusion cuts
        keep = rng.uniform(0.5, 1.0, size=n)
        lo = rng.uniform(0.0, 1.0, size=n) * (1.0 - keep)
        s0 = np.where(occl, lo * length, s0)
        s1 = np.where(occl, (lo + keep) * length, s1)
        return route, off, speed, s0, s1

    def _render(self, route, off, speed, s0, s1, gap, phase, rng):
        """Detections every `gap` native frames starting at `phase`."""
        n = route.shape[0]
        first = s0 + phase * speed
        step = gap * speed
        count = np.maximum(np.floor((s1 - first) / step).astype(np.int64) + 1, 1)
        offsets = np.zeros(n + 1, dtype=np.int64)
        offsets[1:] = np.cumsum(count)
        tid = np.repeat(np.arange(n), count)
        k = np.arange(offsets[-1]) - offsets[tid]
        s = np.minimum(first[tid] + k * step[tid], s1[tid])
        pts = np.empty((offsets[-1], 2))
        for r, (base, cum, normal) in enumerate(self.routes):
            sel = route[tid] == r
            if not sel.any():
                continue
            ss = s[sel]
            j = np.clip(np.searchsorted(cum, ss, side="right") - 1, 0, len(cum) - 2)
            t = ((ss - cum[j]) / np.maximum(cum[j + 1] - cum[j], 1e-12))[:, None]
            p = base[j] + t * (base[j + 1] - base[j])
            nv = normal[j]
            pts[sel] = p + off[tid[sel], None] * nv
        pts += rng.normal(0.0, 0.7 * self.scale, size=pts.shape)
        pts[:, 0] = np.clip(pts[:, 0], 0.0, self.W - 1.0)
        pts[:, 1] = np.clip(pts[:, 1], 0.0, self.H - 1.0)
        return pts.astype(np.float32), offsets

    def _truth(self, route, off, s):
        out = np.empty((route.shape[0], 2))
        for i, (r, o, ss) in enumerate(zip(route, off, s)):
            base, cum, normal = self.routes[r]
            j = int(np.clip(np.searchsorted(cum, ss, side="right") - 1, 0, len(cum) - 2))
            t = (ss - cum[j]) / max(cum[j + 1] - cum[j], 1e-12)
            out[i] = base[j] + t * (base[j + 1] - base[j]) + o * normal[j]
        return out.astype(np.float32)

    def training(self, n: int, seed: int):
        """S*: n tracks at the native frame rate (gap 1)."""
        rng = np.random.Generator(np.random.PCG64(seed))
        route, off, speed, s0, s1 = self._draw(n, rng)
        return self._render(route, off, speed, s0, s1, 1, np.zeros(n), rng)

    def queries(self, n: int, gap: int, seed: int):
        """n tracks captured at gap g -> (points, offsets, true_start [n,2], true_end [n,2], route)."""
        rng = np.random.Generator(np.random.PCG64(seed))
        route, off, speed, s0, s1 = self._draw(n, rng)
        phase = rng.integers(0, gap, size=n).astype(np.float64)
        pts, offsets = self._render(route, off, speed, s0, s1, gap, phase, rng)
        return pts, offsets, self._truth(route, off, s0), self._truth(route, off, s1), route


# C6 (NEXT-4): a 1280x720 junction; S* = 16384 native-rate tracks, 65536 query tracks at g = 16
C6 = TrackWorkload("C6", 1280, 720, n_train=16384, n_query=65536, gap=16, seed=6000)
C6_SMALL = TrackWorkload("C6s", 1280, 720, n_train=600, n_query=256, gap=16, seed=6100, min_pts=4)


def make(wl: TrackWorkload):
    return JunctionScene(wl.width, wl.height, wl.seed)
