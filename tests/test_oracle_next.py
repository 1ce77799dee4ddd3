"""Pins for the oracle's §8(f) NEXT rows: window-size selection (NEXT-1) and
the recall numerator of the proxy-tuning sweep (NEXT-2).  Closed-form cases
(isolated cells, fixed-size clusters), invariants, and hand-made containment cases."""
import numpy as np
import pytest

import oracle

FW, FH, CELL = 416, 256, 32


def masks_with(cells_per_frame, gh=8, gw=13):
    m = np.zeros((len(cells_per_frame), gh, gw), np.uint8)
    for f, cells in enumerate(cells_per_frame):
        for (cy, cx) in cells:
            m[f, cy, cx] = 1
    return m


def test_isolated_cells_pick_smallest_fitting_size():
    # every frame has one isolated cell: 64x64 covers it (cost 4096) -> chosen first;
    # afterwards nothing decreases the sum -> the loop stops with |W| = 2 (reading R19)
    masks = masks_with([[(1, 1)], [(3, 7)], [(6, 12)], []])
    cands = [(128, 128), (64, 64), (256, 256)]
    idx, est = oracle.choose_window_sizes(masks, CELL, FW, FH, cands, k=3)
    assert idx == [-1, 1]
    assert est == [3 * FW * FH, 3 * 64 * 64]


def test_k1_is_full_frame_only():
    masks = masks_with([[(1, 1)], [], [(2, 2), (2, 3)]])
    idx, est = oracle.choose_window_sizes(masks, CELL, FW, FH, [(64, 64)], k=1)
    assert idx == [-1] and est == [2 * FW * FH]   # empty frames cost nothing


def test_cluster_needs_the_larger_size():
    # a 3x3-cell (96x96 px) component: 64x64 cannot cover it, 128x128 can
    cl = [(y, x) for y in range(2, 5) for x in range(4, 7)]
    masks = masks_with([cl, cl])
    idx, est = oracle.choose_window_sizes(masks, CELL, FW, FH, [(64, 64), (128, 128)], k=3)
    assert idx == [-1, 1]
    assert est == [2 * FW * FH, 2 * 128 * 128]


def test_choice_is_monotone_and_bounded():
    rng = np.random.default_rng(4)
    masks = (rng.random((12, 8, 13)) < 0.08).astype(np.uint8)
    cands = [(w, h) for w in (64, 128, 192) for h in (64, 128)]
    idx, est = oracle.choose_window_sizes(masks, CELL, FW, FH, cands, k=4)
    assert idx[0] == -1 and len(set(idx)) == len(idx)
    assert all(a > b for a, b in zip(est, est[1:]))          # every addition strictly decreases Σ est
    assert est[0] == sum(FW * FH for f in range(12) if masks[f].any())
    # Σ est with the chosen W equals the sum of per-frame est under that W
    W = [(FW, FH)] + [cands[i] for i in idx[1:]]
    assert est[-1] == sum(oracle.frame_est(masks[f], CELL, FW, FH, W) for f in range(12))


def test_covered_hand_cases():
    win = np.zeros(3, oracle.WINDOW_DTYPE)
    win[0] = (0, 0, 0, 64, 64, 0)
    win[1] = (0, 64, 0, 64, 64, 0)
    win[2] = (1, 100, 100, 128, 128, 1)
    boxes = np.array([
        [0, 10, 10, 50, 50],      # inside window 0
        [0, 60, 10, 70, 20],      # straddles windows 0 and 1: not covered by one window
        [0, 64, 0, 128, 64],      # exactly window 1 (half-open)
        [1, 100, 100, 228, 228],  # exactly window 2
        [1, 99, 100, 120, 120],   # one pixel left of window 2
        [2, 0, 0, 5, 5],          # frame without windows
    ], np.int32)
    assert oracle.covered(boxes, win) == 3
