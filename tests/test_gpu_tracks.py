"""GPU parity of NEXT-4, track refinement, against the oracle: resampling,
DBSCAN labels/core flags, centres and refined endpoints are compared bit for bit
(readings R21–R25 fix the fp32/fp64 operation order on both sides).  Small sizes are
checked whole; the C6 bench size (16384 S* tracks, 65536 queries) on samples and
properties."""
import numpy as np
import pytest
import torch

import oracle
from synth import tracks

pytestmark = pytest.mark.gpu

otif = pytest.importorskip("paper_conf_sigmod_bastanim22_b200")
from paper_conf_sigmod_bastanim22_b200 import refine  # noqa: E402


def dev(*arrs):
    return [torch.from_numpy(np.ascontiguousarray(a)).cuda() for a in arrs]


def ragged(list_of_tracks):
    pts = np.concatenate([np.asarray(t, np.float32).reshape(-1, 2) for t in list_of_tracks])
    off = np.zeros(len(list_of_tracks) + 1, np.int64)
    off[1:] = np.cumsum([len(t) for t in list_of_tracks])
    return pts, off


@pytest.fixture(scope="module")
def small():
    wl = tracks.C6_SMALL
    sc = tracks.make(wl)
    pts, off = sc.training(wl.n_train, wl.seed + 1)
    q, qo, *_ = sc.queries(wl.n_query, wl.gap, wl.seed + 2)
    return wl, pts, off, q, qo


@pytest.mark.parametrize("npts", [20, 7, 32])
def test_resample_bit_exact(small, npts):
    wl, pts, off, q, qo = small
    for p, o in ((pts, off), (q, qo)):
        P = refine.otif_track_resample(*dev(p, o), npts=npts).cpu().numpy()
        assert np.array_equal(P, oracle.track_resample(p, o, npts))


def test_resample_edge_tracks():
    p, o = ragged([[(5.5, 6.5)], [(1, 2), (1, 2)], [(0, 0), (10, 0), (10, 9)], [(0, 0), (0, 0), (4, 0), (4, 0)],
                   [(1e-3, 2e-3), (1279.5, 719.25), (3.0, 700.0)]])
    P = refine.otif_track_resample(*dev(p, o)).cpu().numpy()
    assert np.array_equal(P, oracle.track_resample(p, o))
    empty = refine.otif_track_resample(*dev(np.zeros((0, 2), np.float32), np.zeros(1, np.int64)))
    assert empty.shape == (0, 20, 2)


@pytest.mark.parametrize("eps,min_pts,npts", [(12.0, 4, 20), (8.0, 3, 20), (24.0, 10, 20), (2.0, 2, 20),
                                              (12.0, 4, 9)])
def test_dbscan_bit_exact(small, eps, min_pts, npts):
    wl, pts, off, *_ = small
    P = oracle.track_resample(pts, off, npts)
    nc, labels, core = oracle.dbscan(P, eps, min_pts)
    g_labels, g_core, g_nc = refine.otif_track_dbscan(*dev(P), eps, min_pts)
    assert int(g_nc.item()) == nc
    assert np.array_equal(g_labels.cpu().numpy(), labels)
    assert np.array_equal(g_core.cpu().numpy().astype(bool), core)


@pytest.mark.parametrize("n", [1, 2, 31, 33, 97])
def test_dbscan_ragged_sizes(small, n):
    wl, pts, off, *_ = small
    P = oracle.track_resample(pts, off)[:n].copy()
    nc, labels, core = oracle.dbscan(P, 12.0, 2)
    g_labels, g_core, g_nc = refine.otif_track_dbscan(*dev(P), 12.0, 2)
    assert int(g_nc.item()) == nc
    assert np.array_equal(g_labels.cpu().numpy(), labels)


def test_centers_and_refine_bit_exact(small):
    wl, pts, off, q, qo = small
    P = oracle.track_resample(pts, off)
    nc, labels, _ = oracle.dbscan(P, 12.0, 4)
    C, sz = oracle.track_centers(P, labels, nc)
    gC, gsz = refine.otif_track_centers(*dev(P, labels), nc)
    assert np.array_equal(gC.cpu().numpy(), C) and np.array_equal(gsz.cpu().numpy(), sz)
    for k, rho in ((10, 0.0), (10, 32.0), (10, 64.0), (1, 32.0), (16, 0.0), (3, 1e9)):
        out, used = oracle.track_refine(q, qo, C, sz, k, rho)
        gout, gused = refine.otif_track_refine(*dev(q, qo), gC, gsz, k, rho)
        assert np.array_equal(gused.cpu().numpy(), used), (k, rho)
        assert np.array_equal(gout.cpu().numpy(), out), (k, rho)


def test_refine_edge_cases():
    base = np.stack([np.linspace(0, 100, 20), np.full(20, 50)], 1).astype(np.float32)
    C = np.stack([base, base + np.float32([0, 3]), base + np.float32([0, 6])])
    sz = np.array([1, 5, 1], np.int32)
    q, qo = ragged([[(30, 53), (60, 53)], [(900, 900), (950, 900)], [(40, 50)]])
    for k, rho in ((10, 20.0), (1, 0.0), (2, 0.0)):
        out, used = oracle.track_refine(q, qo, C, sz, k, rho)
        gout, gused = refine.otif_track_refine(*dev(q, qo, C, sz), k, rho)
        assert np.array_equal(gout.cpu().numpy(), out) and np.array_equal(gused.cpu().numpy(), used)
    # no clusters at all: every track keeps its own endpoints
    gout, gused = refine.otif_track_refine(*dev(q, qo, C[:0], sz[:0]), 10, 0.0)
    assert gused.sum().item() == 0
    assert np.array_equal(gout.cpu().numpy()[:, :2], q[qo[:-1]])


def test_track_index_full_size_sampled():
    """C6 (16384 S* tracks, 65536 queries, the bench launch configuration): core flags
    and labels checked on sampled tracks against fp32 distances from the oracle, the
    DBSCAN invariants on every track, centres bit-exact, refinement bit-exact on a sample."""
    wl = tracks.C6
    sc = tracks.make(wl)
    pts, off = sc.training(wl.n_train, wl.seed + 1)
    q, qo, *_ = sc.queries(wl.n_query, wl.gap, wl.seed + 2)
    idx = refine.TrackIndex.build(*dev(pts, off), wl.eps, wl.min_pts)
    P = oracle.track_resample(pts, off)
    assert np.array_equal(refine.otif_track_resample(*dev(pts, off)).cpu().numpy(), P)
    labels = idx.labels.cpu().numpy()
    core = idx.core.cpu().numpy().astype(bool)
    nc = idx.centers.shape[0]
    rng = np.random.default_rng(0)
    for i in rng.choice(wl.n_train, 48, replace=False):
        d = np.array([oracle.track_distance(P[i], P[j]) for j in range(wl.n_train)], np.float32)
        nb = d <= np.float32(wl.eps)
        assert core[i] == (nb.sum() >= wl.min_pts)
        cn = nb & core
        if core[i]:
            assert np.all(labels[cn] == labels[i])            # one component per cluster
        else:
            assert labels[i] == (labels[cn].min() if cn.any() else -1)
    # cluster ids are ordered by their smallest core member (reading R23)
    firsts = [np.flatnonzero((labels == c) & core)[0] for c in range(nc)]
    assert firsts == sorted(firsts) and nc > 0 and (labels < nc).all()
    C, sz = oracle.track_centers(P, labels, nc)
    assert np.array_equal(idx.centers.cpu().numpy(), C) and np.array_equal(idx.sizes.cpu().numpy(), sz)
    out, used = idx.refine(*dev(q, qo), wl.k, wl.rho)
    sel = rng.choice(wl.n_query, 512, replace=False)
    sub = [q[qo[t]:qo[t + 1]] for t in sel]
    sp, so = ragged(sub)
    o_out, o_used = oracle.track_refine(sp, so, C, sz, wl.k, wl.rho)
    assert np.array_equal(out.cpu().numpy()[sel], o_out)
    assert np.array_equal(used.cpu().numpy()[sel], o_used)
