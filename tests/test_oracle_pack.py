"""Pins for the oracle's crop/pack: pack = crop(resize(src)) with
slots in emission order per size; identity case byte-exact against numpy slicing;
resampling case against OpenCV at an integer factor."""
import numpy as np
import pytest

import oracle
from synth import configs, video

cv2 = pytest.importorskip("cv2")


def _windows(rows):
    w = np.zeros(len(rows), oracle.WINDOW_DTYPE)
    for i, r in enumerate(rows):
        w[i] = r
    return w


def test_identity_pack_is_numpy_crop():
    src = video.frames(configs.C1, 3).numpy()
    sizes = [(64, 64), (128, 128), (416, 256)]
    rows = [(0, 10, 20, 64, 64, 0), (0, 200, 100, 128, 128, 1), (1, 0, 0, 416, 256, 2),
            (2, 352, 192, 64, 64, 0), (2, 1, 3, 64, 64, 0)]
    win = _windows(rows)
    batches, slot, counts = oracle.pack_windows(src, 256, 416, win, sizes)
    assert list(counts) == [3, 1, 1]
    assert list(slot) == [0, 0, 0, 1, 2]
    for g, (f, x, y, w, h, s) in enumerate(rows):
        assert np.array_equal(batches[s][slot[g]], src[f, y:y + h, x:x + w])


def test_pack_with_resample_equals_crop_of_resize():
    src = video.frames(configs.C4_BASE, 2).numpy()       # 1280x720
    det_h, det_w = 360, 640                               # detector at 1/2 (integer factor)
    sizes = [(128, 128), (640, 360)]
    rows = [(0, 5, 7, 128, 128, 0), (1, 0, 0, 640, 360, 1), (1, 512, 232, 128, 128, 0)]
    win = _windows(rows)
    batches, slot, counts = oracle.pack_windows(src, det_h, det_w, win, sizes)
    det = np.stack([cv2.resize(f, (det_w, det_h), interpolation=cv2.INTER_LINEAR) for f in src])
    for g, (f, x, y, w, h, s) in enumerate(rows):
        assert np.array_equal(batches[s][slot[g]], det[f, y:y + h, x:x + w])


def test_pack_capacity_drops_but_counts_exact():
    src = video.frames(configs.C1, 1).numpy()
    sizes = [(64, 64), (416, 256)]
    rows = [(0, 0, 0, 64, 64, 0), (0, 64, 0, 64, 64, 0), (0, 128, 0, 64, 64, 0)]
    batches, slot, counts = oracle.pack_windows(src, 256, 416, _windows(rows), sizes, batch_cap=[2, 0])
    assert list(counts) == [3, 0] and list(slot) == [0, 1, 2]
    assert batches[0].shape[0] == 2
    assert np.array_equal(batches[0][1], src[0, 0:64, 64:128])
