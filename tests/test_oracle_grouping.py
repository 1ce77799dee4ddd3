"""Pins for the oracle's connected components and window grouping (P:L133, P:L149–155,
P:L228; readings R6–R11, R14, R15, R17).

* components: scipy.ndimage.label (library routine) as canonical partitions;
  checkerboard closed forms;
* grouping: invariants on every frame (exact cover, disjointness, in-frame, sizes in W,
  est(R) <= T_full, (y,x) order), brute force over all set partitions of <= 7
  components (est(greedy) >= optimum), and hand-computed special cases.
Beyond these pins the exact greedy output is "parity unpinned" (Fig. 3 is lost).
"""
import itertools

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle

ndi = pytest.importorskip("scipy.ndimage")

W_C1 = [(64, 64), (128, 128), (416, 256)]


def canonical(labels):
    """Relabel by first occurrence in raster order; background -1."""
    out = np.full(labels.shape, -1, np.int64)
    m = {}
    for i, v in enumerate(labels.reshape(-1)):
        if v < 0:
            continue
        if v not in m:
            m[v] = len(m)
        out.reshape(-1)[i] = m[v]
    return out


@pytest.mark.parametrize("conn", [4, 8])
@pytest.mark.parametrize("seed", range(6))
def test_components_match_scipy(conn, seed):
    rng = np.random.default_rng(seed)
    gh, gw = rng.integers(1, 30), rng.integers(1, 45)
    mask = (rng.random((gh, gw)) < rng.uniform(0.1, 0.7)).astype(np.uint8)
    n, lab = oracle.components(mask, conn)
    structure = ndi.generate_binary_structure(2, 1 if conn == 4 else 2)
    ref, nref = ndi.label(mask, structure=structure)
    assert n == nref
    assert np.array_equal(canonical(lab), canonical(np.where(ref > 0, ref, -1)))
    # oracle labels are already in raster order of their seeds
    assert np.array_equal(lab, canonical(lab))


@pytest.mark.parametrize("gh,gw", [(17, 30), (8, 13), (23, 40), (1, 1), (5, 1)])
def test_checkerboard_closed_form(gh, gw):
    mask = ((np.arange(gh)[:, None] + np.arange(gw)[None, :]) % 2 == 0).astype(np.uint8)
    assert oracle.components(mask, 4)[0] == (gh * gw + 1) // 2
    # 8-connectivity joins diagonal neighbours: one component unless the board is a single line
    expect8 = 1 if (gh >= 2 and gw >= 2) or gh * gw == 1 else (gh * gw + 1) // 2
    assert oracle.components(mask, 8)[0] == expect8


def wset(sizes):
    return [(w, h, w * h) for (w, h) in sizes]


def check_invariants(mask, windows, cell, fw, fh, sizes):
    """Every positive cell in exactly one window; windows disjoint, inside the frame,
    sizes in W, est <= T_full, sorted by (y, x)."""
    gh, gw = mask.shape
    cov = np.zeros((fh, fw), np.int32)
    for r in windows:
        assert 0 <= r["x"] and r["x"] + r["w"] <= fw and 0 <= r["y"] and r["y"] + r["h"] <= fh
        s = sizes[r["size_idx"]]
        assert (r["w"], r["h"]) == (s[0], s[1])
        cov[r["y"]:r["y"] + r["h"], r["x"]:r["x"] + r["w"]] += 1
    assert cov.max() <= 1, "windows overlap"
    for cy, cx in zip(*np.nonzero(mask)):
        x0, y0 = cx * cell, cy * cell
        x1, y1 = min(x0 + cell, fw), min(y0 + cell, fh)
        assert (cov[y0:y1, x0:x1] == 1).all(), "positive cell not covered"
    est = sum(sizes[r["size_idx"]][2] for r in windows)
    tfull = min(s[2] for s in sizes if (s[0], s[1]) == (fw, fh))
    assert est <= tfull
    keys = [(int(r["y"]), int(r["x"])) for r in windows]
    assert keys == sorted(keys)
    if mask.sum() == 0:
        assert len(windows) == 0
    else:
        assert len(windows) >= 1
    return est


@settings(max_examples=150, deadline=None)
@given(st.integers(1, 12), st.integers(1, 16), st.floats(0.0, 0.9), st.integers(0, 2 ** 31 - 1),
       st.sampled_from([4, 8]))
def test_grouping_invariants_random(gh, gw, p, seed, conn):
    rng = np.random.default_rng(seed)
    cell = 32
    fw = gw * cell - int(rng.integers(0, cell))
    fh = gh * cell - int(rng.integers(0, cell))
    sizes = [(min(64, fw), min(64, fh)), (min(128, fw), min(128, fh)), (fw, fh)]
    sizes = wset(sizes)
    mask = (rng.random((gh, gw)) < p).astype(np.uint8)
    win = oracle.group_frame(mask, cell, fw, fh, sizes, connectivity=conn)
    check_invariants(mask, win, cell, fw, fh, sizes)


def set_partitions(items):
    if not items:
        yield []
        return
    first, rest = items[0], items[1:]
    for p in set_partitions(rest):
        for i in range(len(p)):
            yield p[:i] + [[first] + p[i]] + p[i + 1:]
        yield [[first]] + p


def brute_force_optimum(mask, cell, fw, fh, sizes):
    """min over all partitions of the components into groups whose placed windows are
    pairwise disjoint, of sum of fit costs; and the full frame."""
    n, lab = oracle.components(mask, 4)
    boxes = []
    for c in range(n):
        ys, xs = np.nonzero(lab == c)
        boxes.append((xs.min() * cell, ys.min() * cell, min((xs.max() + 1) * cell, fw),
                      min((ys.max() + 1) * cell, fh)))
    order = sorted(range(len(sizes)), key=lambda i: (sizes[i][2], sizes[i][0] * sizes[i][1], sizes[i][0], sizes[i][1]))

    def fitw(b):
        rw, rh = b[2] - b[0], b[3] - b[1]
        for i in order:
            if sizes[i][0] >= rw and sizes[i][1] >= rh:
                s = sizes[i]
                x = min(max(b[0] - (s[0] - rw) // 2, 0), fw - s[0])
                y = min(max(b[1] - (s[1] - rh) // 2, 0), fh - s[1])
                return s[2], (x, y, s[0], s[1])

    tfull = min(s[2] for s in sizes if (s[0], s[1]) == (fw, fh))
    best = tfull
    for part in set_partitions(list(range(n))):
        cost, rects = 0, []
        for grp in part:
            bb = (min(boxes[g][0] for g in grp), min(boxes[g][1] for g in grp),
                  max(boxes[g][2] for g in grp), max(boxes[g][3] for g in grp))
            c, r = fitw(bb)
            cost += c
            rects.append(r)
        ok = all(not (a[0] < b[0] + b[2] and b[0] < a[0] + a[2] and a[1] < b[1] + b[3] and b[1] < a[1] + a[3])
                 for a, b in itertools.combinations(rects, 2))
        if ok:
            best = min(best, cost)
    return best, n


def test_brute_force_lower_bound():
    rng = np.random.default_rng(7)
    cell, fw, fh = 32, 256, 192
    sizes = wset([(64, 64), (128, 128), (256, 192)])
    checked = worse = 0
    while checked < 120:
        mask = (rng.random((6, 8)) < rng.uniform(0.05, 0.35)).astype(np.uint8)
        n = oracle.components(mask, 4)[0]
        if n == 0 or n > 7:
            continue
        win = oracle.group_frame(mask, cell, fw, fh, sizes)
        est = check_invariants(mask, win, cell, fw, fh, sizes)
        opt, _ = brute_force_optimum(mask, cell, fw, fh, sizes)
        assert est >= opt
        worse += est > opt
        checked += 1
    # the greedy is an approximation to R* (P:L151): it must hit the optimum most of the time
    assert worse < checked // 3


def win_list(win):
    return [(int(r["x"]), int(r["y"]), int(r["w"]), int(r["h"]), int(r["size_idx"])) for r in win]


def grid(cells, gh=8, gw=13):
    m = np.zeros((gh, gw), np.uint8)
    for (cy, cx) in cells:
        m[cy, cx] = 1
    return m


def test_special_cases_hand_computed():
    """416x256 frame, 32-px cells (8x13 grid), W = {64^2, 128^2, 416x256}, area costs."""
    S = wset(W_C1)
    g = lambda cells: win_list(oracle.group_frame(grid(cells), 32, 416, 256, S))
    # single cell -> cheapest fitting size, centred with floor, clamped
    assert g([(3, 5)]) == [(144, 80, 64, 64, 0)]
    assert g([(0, 0)]) == [(0, 0, 64, 64, 0)]
    assert g([(7, 12)]) == [(352, 192, 64, 64, 0)]
    # two far-apart cells: cheaper apart (union would need the full frame)
    assert g([(0, 0), (0, 12)]) == [(0, 0, 64, 64, 0), (352, 0, 64, 64, 0)]
    # one-cell gap: union needs 128^2 (16384) > 2 x 4096 -> two touching windows
    assert g([(3, 3), (3, 5)]) == [(80, 80, 64, 64, 0), (144, 80, 64, 64, 0)]
    # adjacent cells are one component -> one 64x64 window
    assert g([(3, 3), (3, 4)]) == [(96, 80, 64, 64, 0)]
    # diagonal cells (separate 4-components) whose union fits the same size -> merged
    assert g([(3, 3), (4, 4)]) == [(96, 96, 64, 64, 0)]
    # phase B: clusters whose union costs more, but whose windows overlap -> merged
    # (here the merged cluster needs the full frame)
    assert g([(1, 3), (2, 3), (3, 3), (4, 4), (5, 4)]) == [(0, 0, 416, 256, 2)]
    # dense mask -> full-frame fallback; all-positive -> one full-frame window
    rng = np.random.default_rng(0)
    dense = (rng.random((8, 13)) < 0.6).astype(np.uint8)
    assert win_list(oracle.group_frame(dense, 32, 416, 256, S)) == [(0, 0, 416, 256, 2)]
    assert win_list(oracle.group_frame(np.ones((8, 13), np.uint8), 32, 416, 256, S)) == [(0, 0, 416, 256, 2)]
    # empty mask -> no windows
    assert win_list(oracle.group_frame(np.zeros((8, 13), np.uint8), 32, 416, 256, S)) == []


def test_fallback_is_strict():
    # two 64x64 windows cost 2*4096; full frame 8192 -> tie -> keep the windows
    S = [(64, 64, 4096), (416, 256, 8192)]
    w = win_list(oracle.group_frame(grid([(0, 0), (7, 12)]), 32, 416, 256, S))
    assert w == [(0, 0, 64, 64, 0), (352, 192, 64, 64, 0)]
    S2 = [(64, 64, 4096), (416, 256, 8191)]
    w2 = win_list(oracle.group_frame(grid([(0, 0), (7, 12)]), 32, 416, 256, S2))
    assert w2 == [(0, 0, 416, 256, 1)]


def test_edge_cells_are_clipped():
    # 540 = 16.875 cells of 32: the bottom cell row is 28 px tall (reading R14)
    S = wset([(128, 128), (256, 256), (960, 540)])
    m = np.zeros((17, 30), np.uint8)
    m[16, 29] = 1
    w = win_list(oracle.group_frame(m, 32, 960, 540, S))
    assert w == [(832, 412, 128, 128, 0)]


def test_validation():
    S = wset(W_C1)
    with pytest.raises(ValueError):   # grid does not match frame/cell
        oracle.group_frame(np.zeros((8, 12), np.uint8), 32, 416, 256, S)
    with pytest.raises(ValueError):   # W lacks the full frame
        oracle.group_frame(np.zeros((8, 13), np.uint8), 32, 416, 256, wset([(64, 64)]))
    with pytest.raises(ValueError):   # size larger than the frame
        oracle.group_frame(np.zeros((8, 13), np.uint8), 32, 416, 256, wset(W_C1 + [(512, 512)]))


def test_select_windows_batch_order_and_offsets():
    rng = np.random.default_rng(5)
    masks = (rng.random((6, 8, 13)) < 0.12).astype(np.uint8)
    masks[2] = 0
    S = wset(W_C1)
    win, counts, offs, total = oracle.select_windows(masks, 32, 416, 256, S)
    assert total == counts.sum() == len(win)
    assert list(offs) == list(np.concatenate([[0], np.cumsum(counts)[:-1]]))
    for f in range(6):
        one = oracle.group_frame(masks[f], 32, 416, 256, S, frame_index=f)
        assert win_list(win[offs[f]:offs[f] + counts[f]]) == win_list(one)
        assert (win["frame"][offs[f]:offs[f] + counts[f]] == f).all()
    # capacity overflow: total stays exact
    w2, c2, o2, t2 = oracle.select_windows(masks, 32, 416, 256, S, capacity=2)
    assert t2 == total and len(w2) == min(2, total)


@pytest.mark.parametrize("seed", range(40))
def test_full_fit_cluster_forces_full_frame(seed):
    """The kernel's exact full-frame exit (select.cu): once ANY cluster's minimum-cost
    fitting size is the full frame, the greedy's output is the single full-frame window
    (phase B merges every other cluster into the full-frame placement; R10, R11).  Checked
    on the oracle for masks whose components include one that only the full frame holds."""
    rng = np.random.default_rng(seed)
    fw, fh, cell = 960, 540, 32
    gh, gw = -(-fh // cell), -(-fw // cell)
    sizes = [(128, 128), (256, 256), (fw, fh)]
    mask = (rng.random((gh, gw)) < rng.uniform(0.05, 0.3)).astype(np.uint8)
    # a snake component wider than 256 px (so only the full frame contains it)
    y = int(rng.integers(0, gh))
    x0 = int(rng.integers(0, gw - 10))
    mask[y, x0:x0 + int(rng.integers(9, gw - x0 + 1))] = 1
    n, lab = oracle.components(mask, 4)
    full_fit = False
    for c in range(n):
        ys, xs = np.nonzero(lab == c)
        w = min(int(xs.max() + 1) * cell, fw) - int(xs.min()) * cell
        h = min(int(ys.max() + 1) * cell, fh) - int(ys.min()) * cell
        full_fit |= not any(sw >= w and sh >= h for sw, sh in sizes[:2])
    assert full_fit
    win = oracle.group_frame(mask, cell, fw, fh, sizes)
    assert len(win) == 1
    assert (int(win[0]["x"]), int(win[0]["y"]), int(win[0]["w"]), int(win[0]["h"])) == (0, 0, fw, fh)
