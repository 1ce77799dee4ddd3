"""Pins for the oracle's stage-1 resize (reading R13).

The oracle is checked against things other than itself: OpenCV's INTER_LINEAR and
torch's fp64 bilinear (library routines with the same half-pixel convention),
the closed form of an exact 2x downscale, and invariants.
"""
import numpy as np
import pytest
import torch

import oracle
from synth import configs, video

cv2 = pytest.importorskip("cv2")


def _torch_round(src, h, w):
    t = torch.nn.functional.interpolate(torch.from_numpy(src).permute(0, 3, 1, 2).double(), size=(h, w),
                                        mode="bilinear", align_corners=False, antialias=False)
    return torch.floor(t + 0.5).clamp(0, 255).to(torch.uint8).permute(0, 2, 3, 1).numpy()


@pytest.mark.parametrize("wl,factor", [(configs.C1, 4), (configs.C2, 4), (configs.C4_BASE, 2),
                                       (configs.C4_BASE, 8)])
def test_integer_factor_matches_libraries_exactly(wl, factor):
    src = video.frames(wl, 2).numpy()
    h, w = wl.src_h // factor, wl.src_w // factor
    out = oracle.resize(src, h, w)
    assert np.array_equal(out, _torch_round(src, h, w))
    cv = np.stack([cv2.resize(f, (w, h), interpolation=cv2.INTER_LINEAR) for f in src])
    assert np.array_equal(out, cv)


@pytest.mark.parametrize("h,w", [(256, 416), (187, 333), (540, 960), (77, 131), (1000, 1500)])
def test_non_integer_factor_within_one_lsb(h, w):
    src = video.frames(configs.C4_BASE, 1).numpy()
    out = oracle.resize(src, h, w)
    ref = _torch_round(src, h, w)
    d = np.abs(out.astype(np.int32) - ref)
    assert d.max() <= 1
    assert (d == 0).mean() > 0.95
    cv = cv2.resize(src[0], (w, h), interpolation=cv2.INTER_LINEAR)[None]
    assert np.abs(out.astype(np.int32) - cv).max() <= 1


def test_exact_2x_downscale_is_2x2_mean():
    rng = np.random.default_rng(0)
    src = rng.integers(0, 256, size=(3, 38, 54, 3), dtype=np.uint8)
    out = oracle.resize(src, 19, 27)
    s = src.astype(np.int64)
    mean4 = s[:, 0::2, 0::2] + s[:, 1::2, 0::2] + s[:, 0::2, 1::2] + s[:, 1::2, 1::2]
    expect = (mean4 + 2) // 4  # floor(sum/4 + 0.5)
    assert np.array_equal(out, expect.astype(np.uint8))


@pytest.mark.parametrize("h,w", [(64, 104), (135, 240), (17, 5), (300, 500)])
def test_constant_frame_stays_constant(h, w):
    src = np.full((2, 135, 240, 3), 0, np.uint8)
    src[0] = 37
    src[1, :, :, 0], src[1, :, :, 1], src[1, :, :, 2] = 0, 128, 255
    out = oracle.resize(src, h, w)
    assert (out[0] == 37).all()
    assert (out[1, :, :, 0] == 0).all() and (out[1, :, :, 1] == 128).all() and (out[1, :, :, 2] == 255).all()


def test_same_size_is_exact_copy():
    src = video.frames(configs.C1, 3).numpy()
    assert np.array_equal(oracle.resize(src, configs.C1.src_h, configs.C1.src_w), src)


def test_rejects_bad_sizes():
    src = np.zeros((1, 8, 8, 3), np.uint8)
    with pytest.raises(ValueError):
        oracle.resize(src, 0, 4)
