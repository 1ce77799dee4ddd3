"""CPU oracle for the OTIF proxy + windowing hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_sigmod_bastanim22_b200``) never imports it and shares no code with it.

This module is a thin ctypes binding over ``oracle/otif_ref.c`` (plain C99, fp64,
single-threaded; every function cites the PAPER.md passage it follows).  Arguments
are numpy arrays on the host.

Parity status: resize, conv, threshold, components and pack are pinned by
``tests/test_oracle_*.py``; grouping is pinned by invariants, brute force and
special cases, while its exact greedy output beyond those pins is
"parity unpinned" (PAPER.md's worked example, Fig. 3 at P:L122, is lost).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "otif_ref.c")
_SRCS = [_SRC, os.path.join(_HERE, "otif_ref_tracks.c"), os.path.join(_HERE, "otif_ref_train.c")]

QUANT_NONE = 0
QUANT_BF16 = 1


class WSize(ctypes.Structure):
    _fields_ = [("w", ctypes.c_int32), ("h", ctypes.c_int32), ("cost", ctypes.c_int64)]


class Window(ctypes.Structure):
    _fields_ = [("frame", ctypes.c_int32), ("x", ctypes.c_int32), ("y", ctypes.c_int32),
                ("w", ctypes.c_int32), ("h", ctypes.c_int32), ("size_idx", ctypes.c_int32)]


WINDOW_DTYPE = np.dtype([("frame", "<i4"), ("x", "<i4"), ("y", "<i4"),
                         ("w", "<i4"), ("h", "<i4"), ("size_idx", "<i4")])


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc -O2 (no -ffast-math; -ffp-contract=off so every
    arithmetic operation is one IEEE rounding in the written order)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            [os.path.getmtime(f) for f in _SRCS] + [os.path.getmtime(os.path.join(_HERE, "otif_ref.h"))]):
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-Wall",
                               "-o", _SO] + _SRCS + ["-lm"])
    return _SO


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        P = ctypes.c_void_p
        i32, i64, sz = ctypes.c_int32, ctypes.c_int64, ctypes.c_size_t
        L.otif_ref_round_bf16.argtypes = [ctypes.c_double]
        L.otif_ref_round_bf16.restype = ctypes.c_double
        L.otif_ref_resize.argtypes = [P, i32, i32, i32, P, i32, i32]
        L.otif_ref_conv.argtypes = [P, i32, i32, i32, i32, P, P, i32, i32, i32, i32, i32, P]
        L.otif_ref_proxy_n_weights.argtypes = [P, i32]
        L.otif_ref_proxy_n_weights.restype = sz
        L.otif_ref_proxy_grid.argtypes = [i32, i32, i32, P, P]
        L.otif_ref_proxy_score.argtypes = [P, i32, i32, i32, i32, P, i32, P, sz, i32, P]
        L.otif_ref_threshold.argtypes = [P, i64, ctypes.c_float, P]
        L.otif_ref_components.argtypes = [P, i32, i32, i32, P]
        L.otif_ref_group_frame.argtypes = [P, i32, i32, i32, i32, i32, i32, P, i32, i32, P, i32]
        L.otif_ref_select_windows.argtypes = [P, i32, i32, i32, i32, i32, i32, i32, P, i32,
                                              P, i32, P, P, P]
        L.otif_ref_pack_windows.argtypes = [P, i32, i32, i32, i32, i32, P, i32, P, i32,
                                            P, P, P, P]
    return _lib


def _p(a: np.ndarray) -> ctypes.c_void_p:
    assert a.flags["C_CONTIGUOUS"]
    return ctypes.c_void_p(a.ctypes.data)


def _check(rc: int, what: str) -> int:
    if rc < 0:
        raise ValueError(f"{what}: oracle rejected the arguments (rc={rc})")
    return rc


def wsizes(sizes: Sequence[tuple]) -> ctypes.Array:
    """[(w, h)] or [(w, h, cost)] -> ctypes array; default cost w*h (reading R8)."""
    arr = (WSize * len(sizes))()
    for i, s in enumerate(sizes):
        w, h = int(s[0]), int(s[1])
        arr[i].w, arr[i].h = w, h
        arr[i].cost = int(s[2]) if len(s) > 2 else w * h
    return arr


def round_bf16(x: float) -> float:
    return lib().otif_ref_round_bf16(float(x))


def resize(src: np.ndarray, dh: int, dw: int) -> np.ndarray:
    src = np.ascontiguousarray(src, dtype=np.uint8)
    n, sh, sw, c = src.shape
    assert c == 3
    dst = np.empty((n, dh, dw, 3), np.uint8)
    _check(lib().otif_ref_resize(_p(src), n, sh, sw, _p(dst), dh, dw), "resize")
    return dst


def conv(x: np.ndarray, weight: np.ndarray, bias: np.ndarray, stride: int, relu: bool = True,
         round_bf16_out: bool = False) -> np.ndarray:
    """x [n,h,w,cin] fp64, weight [cout,k,k,cin], bias [cout] -> [n,ceil(h/s),ceil(w/s),cout]."""
    x = np.ascontiguousarray(x, np.float64)
    weight = np.ascontiguousarray(weight, np.float64)
    bias = np.ascontiguousarray(bias, np.float64)
    n, h, w, cin = x.shape
    cout, k, k2, cin2 = weight.shape
    assert k == k2 and cin == cin2
    ho, wo = -(-h // stride), -(-w // stride)
    out = np.empty((n, ho, wo, cout), np.float64)
    _check(lib().otif_ref_conv(_p(x), n, h, w, cin, _p(weight), _p(bias), cout, k, stride,
                               int(relu), int(round_bf16_out), _p(out)), "conv")
    return out


def proxy_n_weights(enc: Sequence[int], dec: int) -> int:
    e = np.ascontiguousarray(enc, np.int32)
    return int(lib().otif_ref_proxy_n_weights(_p(e), dec))


def proxy_grid(in_h: int, in_w: int, n_strided: int) -> tuple[int, int]:
    gh, gw = np.zeros(1, np.int32), np.zeros(1, np.int32)
    _check(lib().otif_ref_proxy_grid(in_h, in_w, n_strided, _p(gh), _p(gw)), "proxy_grid")
    return int(gh[0]), int(gw[0])


def proxy_score(img: np.ndarray, n_strided: int, enc: Sequence[int], dec: int,
                weights: np.ndarray, quant: int = QUANT_BF16) -> np.ndarray:
    img = np.ascontiguousarray(img, np.uint8)
    n, h, w, c = img.shape
    assert c == 3
    weights = np.ascontiguousarray(weights, np.float32)
    e = np.ascontiguousarray(enc, np.int32)
    gh, gw = proxy_grid(h, w, n_strided)
    out = np.empty((n, gh, gw), np.float64)
    _check(lib().otif_ref_proxy_score(_p(img), n, h, w, n_strided, _p(e), dec, _p(weights),
                                      weights.size, quant, _p(out)), "proxy_score")
    return out


def threshold(scores: np.ndarray, b: float) -> np.ndarray:
    scores = np.ascontiguousarray(scores, np.float64)
    mask = np.empty(scores.shape, np.uint8)
    _check(lib().otif_ref_threshold(_p(scores), scores.size, ctypes.c_float(b), _p(mask)),
           "threshold")
    return mask


def components(mask: np.ndarray, connectivity: int = 4) -> tuple[int, np.ndarray]:
    mask = np.ascontiguousarray(mask, np.uint8)
    gh, gw = mask.shape
    labels = np.empty((gh, gw), np.int32)
    n = _check(lib().otif_ref_components(_p(mask), gh, gw, connectivity, _p(labels)),
               "components")
    return n, labels


def group_frame(mask: np.ndarray, cell: int, frame_w: int, frame_h: int, sizes, connectivity=4,
                frame_index: int = 0) -> np.ndarray:
    mask = np.ascontiguousarray(mask, np.uint8)
    gh, gw = mask.shape
    ws = wsizes(sizes)
    cap = gh * gw + 1
    out = np.zeros(cap, WINDOW_DTYPE)
    m = _check(lib().otif_ref_group_frame(_p(mask), gh, gw, cell, frame_w, frame_h, connectivity,
                                          ws, len(sizes), frame_index, _p(out), cap),
               "group_frame")
    return out[:m].copy()


def select_windows(mask: np.ndarray, cell: int, frame_w: int, frame_h: int, sizes,
                   connectivity: int = 4, capacity: int | None = None):
    """mask [n,gh,gw] -> (windows[total], counts[n], offsets[n], total)."""
    mask = np.ascontiguousarray(mask, np.uint8)
    n, gh, gw = mask.shape
    ws = wsizes(sizes)
    if capacity is None:
        capacity = n * ((gh * gw + 1) // 2) if connectivity == 4 else n * (((gh + 1) // 2) * ((gw + 1) // 2))
        capacity = max(capacity, n)
    win = np.zeros(max(capacity, 1), WINDOW_DTYPE)
    counts = np.zeros(n, np.int32)
    offs = np.zeros(n, np.int32)
    total = np.zeros(1, np.int32)
    _check(lib().otif_ref_select_windows(_p(mask), n, gh, gw, cell, frame_w, frame_h, connectivity,
                                         ws, len(sizes), _p(win), capacity, _p(counts), _p(offs),
                                         _p(total)), "select_windows")
    t = int(total[0])
    return win[:min(t, capacity)].copy(), counts, offs, t


def pack_windows(src: np.ndarray, det_h: int, det_w: int, windows: np.ndarray, sizes,
                 batch_cap: Sequence[int] | None = None):
    """-> (batches list of [cap_s,h_s,w_s,3] u8, slot[total], size_count[k])."""
    src = np.ascontiguousarray(src, np.uint8)
    n, sh, sw, _ = src.shape
    windows = np.ascontiguousarray(windows, WINDOW_DTYPE)
    total = windows.shape[0]
    k = len(sizes)
    ws = wsizes(sizes)
    if batch_cap is None:
        batch_cap = [int((windows["size_idx"] == s).sum()) for s in range(k)]
    batches = [np.zeros((max(int(batch_cap[s]), 0), int(sizes[s][1]), int(sizes[s][0]), 3), np.uint8)
               for s in range(k)]
    ptrs = (ctypes.c_void_p * k)(*[b.ctypes.data for b in batches])
    caps = np.ascontiguousarray(batch_cap, np.int32)
    slot = np.zeros(max(total, 1), np.int32)
    counts = np.zeros(k, np.int32)
    _check(lib().otif_ref_pack_windows(_p(src), n, sh, sw, det_h, det_w, _p(windows), total, ws, k,
                                       ptrs, _p(caps), _p(slot), _p(counts)), "pack_windows")
    return batches, slot[:total].copy(), counts


def _lib2():
    L = lib()
    if not getattr(L, "_next_bound", False):
        P, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        L.otif_ref_frame_est.argtypes = [P, i32, i32, i32, i32, i32, i32, P, i32]
        L.otif_ref_frame_est.restype = i64
        L.otif_ref_choose_window_sizes.argtypes = [P, i32, i32, i32, i32, i32, i32, i32, P, i32, i64, i32, P, P]
        L.otif_ref_covered.argtypes = [P, i64, P, i32]
        L.otif_ref_covered.restype = i64
        L._next_bound = True
    return L


def frame_est(mask: np.ndarray, cell: int, frame_w: int, frame_h: int, sizes, connectivity: int = 4) -> int:
    mask = np.ascontiguousarray(mask, np.uint8)
    gh, gw = mask.shape
    return int(_lib2().otif_ref_frame_est(_p(mask), gh, gw, cell, frame_w, frame_h, connectivity, wsizes(sizes),
                                          len(sizes)))


def choose_window_sizes(masks: np.ndarray, cell: int, frame_w: int, frame_h: int, candidates, k: int,
                        full_cost: int | None = None, connectivity: int = 4):
    """NEXT-1 -> (chosen candidate indices with -1 for the full frame, est after each)."""
    masks = np.ascontiguousarray(masks, np.uint8)
    n, gh, gw = masks.shape
    full_cost = frame_w * frame_h if full_cost is None else full_cost
    idx = np.zeros(k, np.int32)
    est = np.zeros(k, np.int64)
    cands = wsizes(candidates)
    nw = _check(_lib2().otif_ref_choose_window_sizes(_p(masks), n, gh, gw, cell, frame_w, frame_h, connectivity,
                                                     cands, len(candidates), full_cost, k, _p(idx), _p(est)),
                "choose_window_sizes")
    return idx[:nw].tolist(), est[:nw].tolist()


def covered(boxes: np.ndarray, windows: np.ndarray) -> int:
    """NEXT-2 recall numerator: boxes int32 [nb, 5] (frame, x0, y0, x1, y1)."""
    boxes = np.ascontiguousarray(boxes, np.int32).reshape(-1, 5)
    windows = np.ascontiguousarray(windows, WINDOW_DTYPE)
    return int(_lib2().otif_ref_covered(_p(boxes), boxes.shape[0], _p(windows), windows.shape[0]))


# --------------------------------------------------------------------------- NEXT-4
def _lib3():
    L = lib()
    if not getattr(L, "_tracks_bound", False):
        P, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float
        L.otif_ref_track_resample.argtypes = [P, P, i64, i32, P]
        L.otif_ref_track_distance.argtypes = [P, P, i32]
        L.otif_ref_track_distance.restype = f32
        L.otif_ref_dbscan.argtypes = [P, i64, i32, f32, i32, P, P]
        L.otif_ref_dbscan.restype = i32
        L.otif_ref_track_centers.argtypes = [P, P, i64, i32, i32, P, P]
        L.otif_ref_track_refine.argtypes = [P, P, i64, i32, P, P, i32, i32, f32, P, P]
        L._tracks_bound = True
    return L


def _tracks_in(pts, offsets):
    pts = np.ascontiguousarray(pts, np.float32).reshape(-1, 2)
    offsets = np.ascontiguousarray(offsets, np.int64)
    return pts, offsets, offsets.shape[0] - 1


def track_resample(pts: np.ndarray, offsets: np.ndarray, npts: int = 20) -> np.ndarray:
    """P:L196 arc-length resampling (reading R21) -> float32 [n, npts, 2]."""
    pts, offsets, n = _tracks_in(pts, offsets)
    out = np.zeros((n, npts, 2), np.float32)
    _check(_lib3().otif_ref_track_resample(_p(pts), _p(offsets), n, npts, _p(out)), "track_resample")
    return out


def track_distance(a: np.ndarray, b: np.ndarray) -> float:
    """P:L196 mean point distance of two resampled tracks [npts, 2] (fp32, reading R22)."""
    a = np.ascontiguousarray(a, np.float32)
    b = np.ascontiguousarray(b, np.float32)
    assert a.shape == b.shape and a.shape[-1] == 2
    return float(_lib3().otif_ref_track_distance(_p(a), _p(b), a.shape[0]))


def dbscan(P: np.ndarray, eps: float, min_pts: int):
    """P:L198 DBSCAN over resampled tracks [n, npts, 2] (reading R23) -> (nc, labels, core)."""
    P = np.ascontiguousarray(P, np.float32)
    n, npts = P.shape[0], P.shape[1]
    labels = np.zeros(n, np.int32)
    core = np.zeros(n, np.uint8)
    nc = _check(_lib3().otif_ref_dbscan(_p(P), n, npts, eps, min_pts, _p(labels), _p(core)), "dbscan")
    return nc, labels, core.astype(bool)


def track_centers(P: np.ndarray, labels: np.ndarray, nc: int):
    """P:L198 cluster centres -> (centers float32 [nc, npts, 2], sizes int32 [nc])."""
    P = np.ascontiguousarray(P, np.float32)
    labels = np.ascontiguousarray(labels, np.int32)
    n, npts = P.shape[0], P.shape[1]
    centers = np.zeros((nc, npts, 2), np.float32)
    sizes = np.zeros(nc, np.int32)
    _check(_lib3().otif_ref_track_centers(_p(P), _p(labels), n, npts, nc, _p(centers), _p(sizes)), "track_centers")
    return centers, sizes


def track_refine(pts: np.ndarray, offsets: np.ndarray, centers: np.ndarray, sizes: np.ndarray, k: int = 10,
                 rho: float = 0.0):
    """P:L200 refinement of query tracks -> (out float32 [m, 4] = start x, y, end x, y; used int32 [m])."""
    pts, offsets, m = _tracks_in(pts, offsets)
    centers = np.ascontiguousarray(centers, np.float32)
    sizes = np.ascontiguousarray(sizes, np.int32)
    nc, npts = centers.shape[0], (centers.shape[1] if centers.ndim == 3 else 20)
    out = np.zeros((m, 4), np.float32)
    used = np.zeros(m, np.int32)
    _check(_lib3().otif_ref_track_refine(_p(pts), _p(offsets), m, npts, _p(centers), _p(sizes), nc, k, rho, _p(out),
                                         _p(used)), "track_refine")
    return out, used


# --------------------------------------------------------------------------- NEXT-3
def _lib4():
    L = lib()
    if not getattr(L, "_train_bound", False):
        P, i32, i64, f64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
        L.otif_ref_cell_labels.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, P]
        L.otif_ref_conv_backward.argtypes = [P, i32, i32, i32, i32, P, i32, i32, i32, P, P, P, P]
        L.otif_ref_proxy_grad.argtypes = [P, i32, i32, i32, i32, P, i32, P, P, P, P]
        L.otif_ref_adam.argtypes = [P, P, P, P, i64, i32, f64, f64, f64, f64]
        L._train_bound = True
    return L


def cell_labels(boxes: np.ndarray, n: int, gh: int, gw: int, cell: int, frame_w: int, frame_h: int) -> np.ndarray:
    """P:L139 training labels -> u8 [n, gh, gw]."""
    boxes = np.ascontiguousarray(boxes, np.int32).reshape(-1, 5)
    out = np.zeros((n, gh, gw), np.uint8)
    _check(_lib4().otif_ref_cell_labels(_p(boxes), boxes.shape[0], n, gh, gw, cell, frame_w, frame_h, _p(out)),
           "cell_labels")
    return out


def conv_backward(x: np.ndarray, weight: np.ndarray, dy: np.ndarray, stride: int, need_dx: bool = True):
    """fp64 conv backward: x [n,h,w,cin], weight [cout,k,k,cin], dy [n,ho,wo,cout] -> (dx, dW, db)."""
    x = np.ascontiguousarray(x, np.float64)
    weight = np.ascontiguousarray(weight, np.float64)
    dy = np.ascontiguousarray(dy, np.float64)
    n, h, w, cin = x.shape
    cout, k = weight.shape[0], weight.shape[1]
    dx = np.zeros_like(x) if need_dx else None
    dW = np.zeros_like(weight)
    db = np.zeros(cout)
    _check(_lib4().otif_ref_conv_backward(_p(x), n, h, w, cin, _p(weight), cout, k, stride, _p(dy),
                                          _p(dx) if need_dx else None, _p(dW), _p(db)), "conv_backward")
    return dx, dW, db


def proxy_grad(img: np.ndarray, n_strided: int, enc, dec: int, weights: np.ndarray, labels: np.ndarray):
    """NEXT-3 one batch -> (mean BCE loss, fp64 gradient blob)."""
    img = np.ascontiguousarray(img, np.uint8)
    n, h, w, _ = img.shape
    weights = np.ascontiguousarray(weights, np.float64)
    labels = np.ascontiguousarray(labels, np.uint8)
    e = np.ascontiguousarray(enc, np.int32)
    grad = np.zeros_like(weights)
    loss = np.zeros(1)
    _check(_lib4().otif_ref_proxy_grad(_p(img), n, h, w, n_strided, _p(e), dec, _p(weights), _p(labels), _p(loss),
                                       _p(grad)), "proxy_grad")
    return float(loss[0]), grad


def adam(w: np.ndarray, m: np.ndarray, v: np.ndarray, g: np.ndarray, t: int, lr: float, b1: float = 0.9,
         b2: float = 0.999, eps: float = 1e-8):
    """Reading R27 Adam step, in place on fp64 arrays."""
    for a in (w, m, v):
        assert a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]
    g = np.ascontiguousarray(g, np.float64)
    _check(_lib4().otif_ref_adam(_p(w), _p(m), _p(v), _p(g), w.size, t, lr, b1, b2, eps), "adam")
