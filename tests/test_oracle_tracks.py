"""Pins for the NEXT-4 oracle, track refinement: closed-form resampling,
an independent np.interp resampler, the distance's metric properties and closed forms,
scikit-learn's DBSCAN on the same distance matrix, numpy means for the centres, and an
independent brute-force refinement (repeat-expansion weighted median)."""
import numpy as np
import pytest

import oracle
from synth import tracks

N = 20


def ragged(list_of_tracks):
    pts = np.concatenate([np.asarray(t, np.float32).reshape(-1, 2) for t in list_of_tracks])
    off = np.zeros(len(list_of_tracks) + 1, np.int64)
    off[1:] = np.cumsum([len(t) for t in list_of_tracks])
    return pts, off


# ----------------------------------------------------------------------------- resample
def test_resample_straight_line_closed_form():
    # polyline along x with L = 19: point i of N = 20 sits exactly at x = i
    pts, off = ragged([[(0, 0), (3, 0), (10, 0), (19, 0)], [(19, 5), (0, 5)], [(7, 0), (7, 19)]])
    P = oracle.track_resample(pts, off, N)
    i = np.arange(N, dtype=np.float32)
    assert np.array_equal(P[0, :, 0], i) and np.array_equal(P[0, :, 1], np.zeros(N))
    assert np.array_equal(P[1, :, 0], 19 - i) and np.array_equal(P[1, :, 1], np.full(N, 5))
    assert np.array_equal(P[2, :, 1], i) and np.array_equal(P[2, :, 0], np.full(N, 7))


def test_resample_corner_closed_form():
    # L-shaped path (0,0) -> (10,0) -> (10,9): arc length 19, the corner at s = 10
    pts, off = ragged([[(0, 0), (10, 0), (10, 9)]])
    P = oracle.track_resample(pts, off, N)[0]
    want = np.array([(i, 0) if i <= 10 else (10, i - 10) for i in range(N)], np.float32)
    assert np.array_equal(P, want)


def test_resample_degenerate_tracks():
    pts, off = ragged([[(5.5, 6.5)], [(1, 2), (1, 2), (1, 2)], [(0, 0), (0, 0), (4, 0)]])
    P = oracle.track_resample(pts, off, N)
    assert np.all(P[0] == np.float32([5.5, 6.5]))        # one detection: repeated
    assert np.all(P[1] == np.float32([1, 2]))            # zero length: repeated
    # a repeated first point (zero-length segment) is skipped: evenly spaced on (0,0)-(4,0)
    assert np.allclose(P[2, :, 0], 4 * np.arange(N) / (N - 1), atol=1e-6)


def np_interp_resample(p, n=N):
    """Independent resampler: fp64 cumulative arc length + np.interp (not the oracle's code)."""
    p = p.astype(np.float64)
    cum = np.concatenate([[0.0], np.cumsum(np.hypot(*np.diff(p, axis=0).T))])
    if cum[-1] == 0:
        return np.repeat(p[:1], n, 0)
    s = cum[-1] * np.arange(n) / (n - 1)
    return np.stack([np.interp(s, cum, p[:, 0]), np.interp(s, cum, p[:, 1])], 1)


def test_resample_matches_np_interp_on_synthetic_tracks():
    wl = tracks.C6_SMALL
    sc = tracks.make(wl)
    pts, off = sc.training(200, 11)
    q, qo, *_ = sc.queries(200, wl.gap, 12)
    for p, o in ((pts, off), (q, qo)):
        P = oracle.track_resample(p, o, N)
        for t in range(len(o) - 1):
            ref = np_interp_resample(p[o[t]:o[t + 1]])
            assert np.max(np.abs(P[t] - ref)) < 2e-3          # fp32 output of 1280-px values
            assert np.array_equal(P[t, 0], p[o[t]]) and np.array_equal(P[t, -1], p[o[t + 1] - 1])


def test_resample_spacing_is_even():
    rng = np.random.default_rng(3)
    p = np.cumsum(rng.uniform(-5, 5, size=(50, 2)), axis=0).astype(np.float32) + 500
    P = oracle.track_resample(p, np.array([0, 50]), N)[0].astype(np.float64)
    pp = p.astype(np.float64)
    cum = np.concatenate([[0.0], np.cumsum(np.hypot(*np.diff(pp, axis=0).T))])
    # arc-length position of each output point on the polyline is L*i/(N-1)
    for i in range(1, N - 1):
        j = np.searchsorted(cum, cum[-1] * i / (N - 1)) - 1
        pos = cum[j] + np.hypot(*(P[i] - pp[j]))
        assert abs(pos - cum[-1] * i / (N - 1)) < 1e-3


# ----------------------------------------------------------------------------- distance
def test_distance_closed_forms_and_metric():
    a = np.stack([np.arange(N), np.zeros(N)], 1).astype(np.float32)
    assert oracle.track_distance(a, a) == 0.0
    assert oracle.track_distance(a, a + np.float32([3, 4])) == 5.0      # constant offset (3,4)
    b = a.copy()
    b[5] += np.float32([6, 8])                                          # one point off by 10
    assert oracle.track_distance(a, b) == pytest.approx(10 / N, rel=1e-7)
    rng = np.random.default_rng(5)
    T = rng.uniform(0, 1280, size=(12, N, 2)).astype(np.float32)
    for i in range(12):
        for j in range(12):
            dij = oracle.track_distance(T[i], T[j])
            assert dij == oracle.track_distance(T[j], T[i])            # bitwise symmetric
            ref = np.mean(np.hypot(*(T[i].astype(np.float64) - T[j]).T))
            assert dij == pytest.approx(ref, rel=2e-6)
            for k in range(0, 12, 5):
                assert dij <= oracle.track_distance(T[i], T[k]) + oracle.track_distance(T[k], T[j]) + 1e-3


# ----------------------------------------------------------------------------- DBSCAN
def fp32_distance_matrix(P):
    """Input for scikit-learn: mean point distance evaluated in fp32 in index order
    (the decision precision of reading R22), vectorised over pairs."""
    s = np.zeros((P.shape[0], P.shape[0]), np.float32)
    for i in range(P.shape[1]):
        dx = P[:, None, i, 0] - P[None, :, i, 0]
        dy = P[:, None, i, 1] - P[None, :, i, 1]
        s = s + np.sqrt(dx * dx + dy * dy)
    return s / np.float32(P.shape[1])


@pytest.mark.parametrize("eps,min_pts", [(12.0, 4), (8.0, 3), (24.0, 10), (2.0, 2)])
def test_dbscan_matches_sklearn(eps, min_pts):
    from sklearn.cluster import DBSCAN
    wl = tracks.C6_SMALL
    pts, off = tracks.make(wl).training(400, 21)
    P = oracle.track_resample(pts, off, N)
    nc, labels, core = oracle.dbscan(P, eps, min_pts)
    D = fp32_distance_matrix(P)
    # spot-check the vectorised matrix against the oracle's own distance
    for i, j in ((0, 1), (5, 399), (123, 7)):
        assert D[i, j] == oracle.track_distance(P[i], P[j])
    sk = DBSCAN(eps=eps, min_samples=min_pts, metric="precomputed").fit(D.astype(np.float64))
    assert np.array_equal(labels, sk.labels_)
    assert np.array_equal(np.flatnonzero(core), np.sort(sk.core_sample_indices_))
    assert nc == sk.labels_.max() + 1


def test_dbscan_special_cases():
    # two tight groups far apart + one isolated track; min_pts 3
    base = np.stack([np.arange(N), np.zeros(N)], 1).astype(np.float32)
    P = np.stack([base, base + 1, base + 2, base + 500, base + 501, base + 502, base + 250])
    nc, labels, core = oracle.dbscan(P, 3.0, 3)
    assert nc == 2 and labels.tolist() == [0, 0, 0, 1, 1, 1, -1]
    # a border track X between two clusters joins the earlier-numbered one (reading R23):
    # x-offsets X=5 (index 0), B = {8, 10 x4} (indices 1-5, cluster 0), A = {0 x4, 2}
    # (cluster 1); eps 3, min_pts 5: N(X) = {X, 2, 8} -> border of both, label 0
    offs = [5, 8, 10, 10, 10, 10, 0, 0, 0, 0, 2]
    Q = np.stack([base + np.float32([o, 0]) for o in offs])
    nc, labels, core = oracle.dbscan(Q, 3.0, 5)
    assert nc == 2 and not core[0] and core[1:].all()
    assert labels.tolist() == [0] + [0] * 5 + [1] * 5
    nc, labels, core = oracle.dbscan(np.zeros((0, N, 2), np.float32), 1.0, 2)
    assert nc == 0 and labels.shape == (0,)


# ----------------------------------------------------------------------------- centres
def test_centers_are_member_means():
    wl = tracks.C6_SMALL
    pts, off = tracks.make(wl).training(300, 31)
    P = oracle.track_resample(pts, off, N)
    nc, labels, _ = oracle.dbscan(P, 12.0, 4)
    C, sz = oracle.track_centers(P, labels, nc)
    assert nc > 2
    assert np.array_equal(sz, np.bincount(labels[labels >= 0], minlength=nc))
    for c in range(nc):
        ref = P[labels == c].astype(np.float64).mean(0)
        assert np.max(np.abs(C[c] - ref)) < 1e-4


# ----------------------------------------------------------------------------- refine
def brute_refine(q, qo, C, sz, k, rho):
    """Independent refinement: numpy distances, lexsort kNN, repeat-expansion medians."""
    Pq = oracle.track_resample(q, qo, C.shape[1]) if len(qo) > 1 else np.zeros((0, C.shape[1], 2), np.float32)
    out = np.zeros((len(qo) - 1, 4), np.float32)
    used = np.zeros(len(qo) - 1, np.int32)
    for t in range(len(qo) - 1):
        d1, dn = q[qo[t]], q[qo[t + 1] - 1]
        s = np.zeros(len(C), np.float32)
        for i in range(C.shape[1]):
            dx, dy = Pq[t, i, 0] - C[:, i, 0], Pq[t, i, 1] - C[:, i, 1]
            s = s + np.sqrt(dx * dx + dy * dy)
        d = s / np.float32(C.shape[1])
        ok = np.ones(len(C), bool)
        if rho > 0:
            near = lambda p: (np.sqrt((C[:, :, 0] - p[0]) ** 2 + (C[:, :, 1] - p[1]) ** 2) <= np.float32(rho)).any(1)
            ok = near(d1) & near(dn)
        idx = np.flatnonzero(ok)
        idx = idx[np.lexsort((idx, d[idx]))][:k]
        used[t] = len(idx)
        if len(idx) == 0:
            out[t] = [d1[0], d1[1], dn[0], dn[1]]
            continue
        for e, (pi, ci) in enumerate(((0, 0), (0, 1), (-1, 0), (-1, 1))):
            expanded = np.sort(np.repeat(C[idx, pi, ci], sz[idx]))
            out[t, e] = expanded[(int(sz[idx].sum()) + 1) // 2 - 1]
    return out, used


@pytest.mark.parametrize("rho", [0.0, 32.0, 64.0])
def test_refine_matches_brute_force(rho):
    wl = tracks.C6_SMALL
    sc = tracks.make(wl)
    pts, off = sc.training(wl.n_train, wl.seed + 1)
    P = oracle.track_resample(pts, off, N)
    nc, labels, _ = oracle.dbscan(P, 12.0, 4)
    C, sz = oracle.track_centers(P, labels, nc)
    q, qo, *_ = sc.queries(120, wl.gap, wl.seed + 2)
    out, used = oracle.track_refine(q, qo, C, sz, 10, rho)
    bout, bused = brute_refine(q, qo, C, sz, 10, rho)
    assert np.array_equal(used, bused)
    assert np.array_equal(out, bout)


def test_refine_special_cases():
    base = np.stack([np.linspace(0, 100, N), np.full(N, 50)], 1).astype(np.float32)
    C = np.stack([base, base + np.float32([0, 3]), base + np.float32([0, 6])])
    sz = np.array([1, 5, 1], np.int32)
    q, qo = ragged([[(30, 53), (60, 53)], [(900, 900), (950, 900)]])
    out, used = oracle.track_refine(q, qo, C, sz, k=10, rho=20.0)
    # track 0: all three centres pass close; the size-5 middle centre is the weighted median
    assert used[0] == 3 and np.array_equal(out[0], np.float32([0, 53, 100, 53]))
    # track 1: no centre passes close -> keeps its own first/last detection
    assert used[1] == 0 and np.array_equal(out[1], np.float32([900, 900, 950, 900]))
    out, used = oracle.track_refine(q, qo, C, sz, k=1, rho=0.0)
    assert used.tolist() == [1, 1] and np.array_equal(out[0], np.float32([0, 53, 100, 53]))


def test_refinement_reduces_endpoint_error():
    """The method's purpose (Fig. 4): refined start/end are closer to the truth
    than the first/last detection of a gap-16 track, on the synthetic junction."""
    wl = tracks.C6_SMALL
    sc = tracks.make(wl)
    pts, off = sc.training(1500, 41)
    P = oracle.track_resample(pts, off, N)
    nc, labels, _ = oracle.dbscan(P, 12.0, 4)
    C, sz = oracle.track_centers(P, labels, nc)
    q, qo, ts, te, _ = sc.queries(300, wl.gap, 42)
    out, used = oracle.track_refine(q, qo, C, sz, 10, 32.0)
    raw = np.stack([q[qo[:-1]], q[qo[1:] - 1]], 1)
    err_raw = np.hypot(*(raw[:, 0] - ts).T).mean() + np.hypot(*(raw[:, 1] - te).T).mean()
    err_ref = np.hypot(*(out[:, :2] - ts).T).mean() + np.hypot(*(out[:, 2:] - te).T).mean()
    assert used.mean() > 0.5
    assert err_ref < 0.8 * err_raw
