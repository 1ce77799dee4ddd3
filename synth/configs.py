"""Workload definitions C1–C5 (BASELINE.json "configs").

Plain data: sizes, seeds and window-size sets.  No arithmetic of the method lives
here (the grid shape, strides and windows are computed by the oracle and by the
CUDA library independently).
"""
from __future__ import annotations

import dataclasses
from fractions import Fraction

# Proxy CNN widths, reading R2 (PAPER.md P:L135 gives only the layer counts).
ENC_WIDTHS = (32, 64, 128, 256, 256)
DEC_WIDTH = 128
WEIGHT_SEED = 20220612  # reading R3


@dataclasses.dataclass(frozen=True)
class Workload:
    name: str
    scene: str              # "traffic" (fixed camera) or "uav" (moving camera)
    src_w: int
    src_h: int
    n_frames: int
    proxy_scale: Fraction   # r: proxy input = r * source
    cell: int               # c: cell size in detector pixels (reading R1)
    sizes: tuple            # W as ((w, h), ...); cost defaults to w*h
    seed: int
    quantile: float = 0.7   # reading R5
    gap: int = 4            # sampling gap g
    objects: float = 10.0   # traffic scenes: mean concurrent objects at 960x540

    @property
    def proxy_w(self) -> int:
        v = self.src_w * self.proxy_scale
        assert v.denominator == 1
        return int(v)

    @property
    def proxy_h(self) -> int:
        v = self.src_h * self.proxy_scale
        assert v.denominator == 1
        return int(v)

    @property
    def stride(self) -> int:
        """S = c * r, the proxy's output stride (reading R1)."""
        v = self.cell * self.proxy_scale
        assert v.denominator == 1
        return int(v)

    @property
    def n_strided(self) -> int:
        s = self.stride
        assert s & (s - 1) == 0 and 2 <= s <= 32
        return s.bit_length() - 1

    def with_(self, **kw) -> "Workload":
        return dataclasses.replace(self, **kw)


C1 = Workload("C1", "traffic", 416, 256, 32, Fraction(1, 4), 32,
              ((64, 64), (128, 128), (416, 256)), seed=1000)
C2 = Workload("C2", "traffic", 960, 540, 4500, Fraction(1, 4), 32,
              ((128, 128), (256, 256), (960, 540)), seed=2000)
# C2 at off-peak density (~4 concurrent vehicles instead of ~13): the same camera, the
# regime in which windows beat the full frame
C2S = C2.with_(name="C2s", objects=3.0)
C3 = Workload("C3", "uav", 1920, 1080, 3000, Fraction(1, 4), 64,
              ((64, 64), (128, 128), (256, 256), (512, 512), (1920, 1080)), seed=3000, gap=1)
C4_BASE = Workload("C4", "traffic", 1280, 720, 450, Fraction(1, 4), 32,
                   ((128, 128), (256, 256), (1280, 720)), seed=4000)
# the joint-tuning grid: proxy resolution x cell size (x threshold quantile)
C4_SWEEP = tuple(
    C4_BASE.with_(name=f"C4{tag}", proxy_scale=r, cell=c)
    for tag, r, c in (("a", Fraction(1, 2), 32), ("b", Fraction(1, 4), 32), ("c", Fraction(1, 8), 32),
                      ("d", Fraction(1, 2), 64), ("e", Fraction(1, 4), 64), ("f", Fraction(1, 8), 64)))
C4_QUANTILES = (0.5, 0.7, 0.8, 0.9)
# 8 h of 960x540 = 480 one-minute clips x 450 sampled frames
C5 = C2.with_(name="C5", n_frames=216000, seed=5000)
C5_CLIPS = 480
C5_FRAMES_PER_CLIP = 450
C5_POOL_CLIPS = 8

ALL = {w.name: w for w in (C1, C2, C2S, C3, C5) + C4_SWEEP}
